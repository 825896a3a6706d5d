/*
 * oracle/oracle.c — CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_eurosys_0002a0a024_b200/) never imports, links or executes it; the two
 * trees share no code, headers, tables or helpers.
 *
 * Plain, slow, obviously-correct implementations of what the Core Graph
 * hot path computes, each citing the passage of /root/reference/PAPER.md
 * ("P:<line>") it follows.  Readings of garbled / ambiguous passages are
 * the SURVEY.md §8(c) readings Q1..Q20, listed in DESIGN.md.
 *
 *  - or_canonical_csr / or_transpose: the graph G(V,E) as CSR,
 *    and its reverse G^R(V,E^R) (Alg 1 l.5 P:741, Alg 2 l.7 P:1043).
 *    Canonical form (reading Q14): self-loops dropped, parallel edges
 *    collapsed to the minimum weight, rows sorted by destination.
 *  - or_query: the vertex-specific query definition: Val(v) =
 *    select over all s->v paths of the fold of (+) from SourceInitVal, with
 *    the per-kind operators of Table 6.  Because every (+) is
 *    non-improving and monotone, a label-setting Dijkstra
 *    with the kind's priority IS that definition; it is pinned against
 *    brute-force path enumeration in tests/.
 *  - or_bellman_ford: synchronous (Jacobi) fixpoint of the same relaxation,
 *    an independent cross-check.
 *  - or_hubs_topdeg: "20 highest degree vertices",
 *    reading Q7 (total degree, ties to the smaller id).
 *  - or_cg_alg1: Algorithm 1 literally, incl. the connectivity
 *    edges of l.8-12 (reading Q8).
 *  - or_cg_alg2: Algorithm 2 literally, sequential FIFO with a
 *    shared Qid[] (readings Q9-Q11).
 *  - or_2phase / or_full_bsp: Algorithm 3 literally in
 *    sequential BSP order (readings Q1-Q5).
 *  - or_wcc: weakly connected components (NEXT-3, Table 6 WCC row): the
 *    minimum vertex id of each weak component, by union-find.
 *  - or_certified: O7, the precision certificates of the Reduced(E)
 *    optimization (NEXT-1): Theorem 1 for SSSP / BFS, its
 *    bottleneck analogs for SSWP / SSNP, the lattice top for REACH.
 *
 * Value words: every kind stores a 32-bit word per vertex; Viterbi stores
 * the IEEE-754 binary32 bit pattern (reading Q13: f32, RN division).
 * Kind numbering: 0 SSSP, 1 SSWP, 2 SSNP, 3 VITERBI, 4 BFS, 5 REACH.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { K_SSSP = 0, K_SSWP = 1, K_SSNP = 2, K_VITERBI = 3, K_BFS = 4, K_REACH = 5, K_NKINDS = 6 };

/* ------------------------------------------------------------------ */
/* Per-kind operators: Table 6 + reading Q1 init values.  */
/* ------------------------------------------------------------------ */

static float w2f(uint32_t x) { float f; memcpy(&f, &x, 4); return f; }
static uint32_t f2w(float f) { uint32_t x; memcpy(&x, &f, 4); return x; }

/* InitVal: the value of an unreached vertex (Alg 3 l.6). */
uint32_t or_init_val(int kind) {
    switch (kind) {
    case K_SSSP: case K_SSNP: case K_BFS: return 0xFFFFFFFFu;  /* +inf */
    case K_SSWP: return 0u;                                     /* width 0 */
    case K_VITERBI: return f2w(0.0f);                            /* probability 0 */
    case K_REACH: return 0u;                                     /* unreached */
    }
    return 0;
}

/* SourceInitVal: the value of the source (Alg 3 l.4). */
uint32_t or_source_val(int kind) {
    switch (kind) {
    case K_SSSP: case K_SSNP: case K_BFS: return 0u;
    case K_SSWP: return 0xFFFFFFFFu;
    case K_VITERBI: return f2w(1.0f);
    case K_REACH: return 1u;
    }
    return 0;
}

/* Val(u) (+) w(u,v): the propagation operator of each kind (Table 6). */
uint32_t or_extend(int kind, uint32_t a, uint32_t w) {
    switch (kind) {
    case K_SSSP: {                                   /* Val(u) + wt(u,v) */
        uint64_t s = (uint64_t)a + (uint64_t)w;
        return s >= 0xFFFFFFFFull ? 0xFFFFFFFEu : (uint32_t)s;  /* saturate below +inf */
    }
    case K_SSWP: return a < w ? a : w;               /* min(Val(u), wt(u,v)) */
    case K_SSNP: return a > w ? a : w;               /* max(Val(u), wt(u,v)) */
    case K_VITERBI: {                                /* Val(u) / wt(u,v), binary32 RN */
        volatile float q = w2f(a) / (float)w;
        return f2w(q);
    }
    case K_BFS: return a + 1u;                       /* hop count */
    case K_REACH: return a;                          /* Val(u) */
    }
    return a;
}

/* a strictly better than b under the kind's selection operator (MIN or MAX). */
int or_better(int kind, uint32_t a, uint32_t b) {
    switch (kind) {
    case K_SSSP: case K_SSNP: case K_BFS: return a < b;   /* MIN */
    case K_SSWP: case K_REACH: return a > b;              /* MAX */
    case K_VITERBI: return w2f(a) > w2f(b);               /* MAX over probabilities */
    }
    return 0;
}

static int reached(int kind, uint32_t x) { return x != or_init_val(kind); }

/* ------------------------------------------------------------------ */
/* Graph construction (reading Q14).                        */
/* ------------------------------------------------------------------ */

typedef struct { uint32_t d, w; } dw_t;

static int cmp_dw(const void* pa, const void* pb) {
    const dw_t* a = (const dw_t*)pa;
    const dw_t* b = (const dw_t*)pb;
    if (a->d != b->d) return a->d < b->d ? -1 : 1;
    if (a->w != b->w) return a->w < b->w ? -1 : 1;
    return 0;
}

/*
 * Canonical CSR of the edge list: bucket by source, sort each row by
 * (dst, w), drop self-loops, keep the first (= minimum-weight) copy of each
 * (src, dst).  row_ptr has n+1 entries; col/wt need capacity m.  Returns the
 * canonical edge count.
 */
int64_t or_canonical_csr(int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst,
                         const uint32_t* w, int64_t* row_ptr, uint32_t* col, uint32_t* wt) {
    int64_t* cnt = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    for (int64_t i = 0; i < m; ++i)
        if (src[i] != dst[i]) cnt[src[i] + 1]++;
    for (int64_t v = 0; v < n; ++v) cnt[v + 1] += cnt[v];
    dw_t* buf = (dw_t*)malloc(sizeof(dw_t) * (size_t)(cnt[n] > 0 ? cnt[n] : 1));
    int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
    memcpy(fill, cnt, sizeof(int64_t) * (size_t)(n + 1));
    for (int64_t i = 0; i < m; ++i) {
        if (src[i] == dst[i]) continue;
        dw_t e = {dst[i], w[i]};
        buf[fill[src[i]]++] = e;
    }
    int64_t out = 0;
    row_ptr[0] = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t b = cnt[v], e = cnt[v + 1];
        qsort(buf + b, (size_t)(e - b), sizeof(dw_t), cmp_dw);
        for (int64_t i = b; i < e; ++i) {
            if (i > b && buf[i].d == buf[i - 1].d) continue;  /* duplicate: keep min w */
            col[out] = buf[i].d;
            wt[out] = buf[i].w;
            ++out;
        }
        row_ptr[v + 1] = out;
    }
    free(cnt);
    free(buf);
    free(fill);
    return out;
}

/* Reverse graph G^R as CSR over reversed edges (= CSC of G); rows sorted by source id. */
void or_transpose(int64_t n, const int64_t* row_ptr, const uint32_t* col, const uint32_t* wt,
                  int64_t* col_ptr, uint32_t* row, uint32_t* wt_t) {
    int64_t m = row_ptr[n];
    memset(col_ptr, 0, sizeof(int64_t) * (size_t)(n + 1));
    for (int64_t i = 0; i < m; ++i) col_ptr[col[i] + 1]++;
    for (int64_t v = 0; v < n; ++v) col_ptr[v + 1] += col_ptr[v];
    int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
    memcpy(fill, col_ptr, sizeof(int64_t) * (size_t)(n + 1));
    for (int64_t u = 0; u < n; ++u)
        for (int64_t i = row_ptr[u]; i < row_ptr[u + 1]; ++i) {
            int64_t p = fill[col[i]]++;
            row[p] = (uint32_t)u;
            wt_t[p] = wt[i];
        }
    free(fill);
}

/* ------------------------------------------------------------------ */
/* Query definition via label-setting Dijkstra.            */
/* ------------------------------------------------------------------ */

typedef struct { uint32_t val; uint32_t v; } hent_t;
typedef struct { hent_t* a; int64_t size, cap; int kind; } heap_t;

/* heap order: "better" value first; ties by smaller vertex id (any order is correct) */
static int hless(const heap_t* h, hent_t x, hent_t y) {
    if (or_better(h->kind, x.val, y.val)) return 1;
    if (or_better(h->kind, y.val, x.val)) return 0;
    return x.v < y.v;
}

static void hpush(heap_t* h, hent_t e) {
    if (h->size == h->cap) {
        h->cap = h->cap ? h->cap * 2 : 1024;
        h->a = (hent_t*)realloc(h->a, sizeof(hent_t) * (size_t)h->cap);
    }
    int64_t i = h->size++;
    h->a[i] = e;
    while (i > 0) {
        int64_t p = (i - 1) / 2;
        if (!hless(h, h->a[i], h->a[p])) break;
        hent_t t = h->a[i]; h->a[i] = h->a[p]; h->a[p] = t;
        i = p;
    }
}

static hent_t hpop(heap_t* h) {
    hent_t top = h->a[0];
    h->a[0] = h->a[--h->size];
    int64_t i = 0;
    for (;;) {
        int64_t l = 2 * i + 1, r = l + 1, b = i;
        if (l < h->size && hless(h, h->a[l], h->a[b])) b = l;
        if (r < h->size && hless(h, h->a[r], h->a[b])) b = r;
        if (b == i) break;
        hent_t t = h->a[i]; h->a[i] = h->a[b]; h->a[b] = t;
        i = b;
    }
    return top;
}

/*
 * Q(s).Val(*) on the graph (ptr, adj, wt).  BFS ignores weights
 * (every edge counts 1).  out has n entries.  Returns the number of edges
 * scanned (for timing context only).
 */
int64_t or_query(int kind, int64_t n, const int64_t* ptr, const uint32_t* adj, const uint32_t* wt,
                 uint32_t s, uint32_t* out) {
    const uint32_t INIT = or_init_val(kind);
    for (int64_t v = 0; v < n; ++v) out[v] = INIT;
    out[s] = or_source_val(kind);
    uint8_t* done = (uint8_t*)calloc((size_t)n, 1);
    heap_t h = {NULL, 0, 0, kind};
    hent_t e0 = {out[s], s};
    hpush(&h, e0);
    int64_t scanned = 0;
    while (h.size > 0) {
        hent_t e = hpop(&h);
        uint32_t u = e.v;
        if (done[u] || e.val != out[u]) continue;  /* stale entry */
        done[u] = 1;
        for (int64_t i = ptr[u]; i < ptr[u + 1]; ++i) {
            uint32_t v = adj[i];
            uint32_t cand = or_extend(kind, out[u], kind == K_BFS ? 1u : wt[i]);
            ++scanned;
            if (!done[v] && or_better(kind, cand, out[v])) {
                out[v] = cand;
                hent_t ne = {cand, v};
                hpush(&h, ne);
            }
        }
    }
    free(h.a);
    free(done);
    return scanned;
}

/* Many sources, one source per OpenMP thread (SURVEY §8(d) "Oracle timing"). */
int64_t or_query_batch(int kind, int64_t n, const int64_t* ptr, const uint32_t* adj,
                       const uint32_t* wt, int64_t nsrc, const uint32_t* srcs, uint32_t* out,
                       int nthreads) {
    int64_t total = 0;
    #pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads) reduction(+ : total)
    for (int64_t q = 0; q < nsrc; ++q)
        total += or_query(kind, n, ptr, adj, wt, srcs[q], out + q * n);
    return total;
}

/*
 * Synchronous (Jacobi) Bellman-Ford fixpoint: round r relaxes every edge
 * out of every reached vertex using round r-1's values.  Returns rounds.
 */
int64_t or_bellman_ford(int kind, int64_t n, const int64_t* ptr, const uint32_t* adj,
                        const uint32_t* wt, uint32_t s, uint32_t* out) {
    const uint32_t INIT = or_init_val(kind);
    uint32_t* prev = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)n);
    for (int64_t v = 0; v < n; ++v) out[v] = INIT;
    out[s] = or_source_val(kind);
    int64_t rounds = 0;
    for (;;) {
        memcpy(prev, out, sizeof(uint32_t) * (size_t)n);
        int changed = 0;
        for (int64_t u = 0; u < n; ++u) {
            if (!reached(kind, prev[u])) continue;
            for (int64_t i = ptr[u]; i < ptr[u + 1]; ++i) {
                uint32_t cand = or_extend(kind, prev[u], kind == K_BFS ? 1u : wt[i]);
                if (or_better(kind, cand, out[adj[i]])) { out[adj[i]] = cand; changed = 1; }
            }
        }
        ++rounds;
        if (!changed) break;
    }
    free(prev);
    return rounds;
}

/* ------------------------------------------------------------------ */
/* Hub selection (reading Q7).     */
/* ------------------------------------------------------------------ */

void or_hubs_topdeg(int64_t n, const int64_t* ptr, const int64_t* cptr, int32_t K, uint32_t* hubs) {
    uint8_t* taken = (uint8_t*)calloc((size_t)n, 1);
    for (int32_t k = 0; k < K; ++k) {
        int64_t best = -1, bestdeg = -1;
        for (int64_t v = 0; v < n; ++v) {
            if (taken[v]) continue;
            int64_t deg = (ptr[v + 1] - ptr[v]) + (cptr[v + 1] - cptr[v]);
            if (deg > bestdeg) { bestdeg = deg; best = v; }  /* strict: ties keep smaller id */
        }
        taken[best] = 1;
        hubs[k] = (uint32_t)best;
    }
    free(taken);
}

/* position of edge (u -> v) in G's CSR (rows sorted by dst), or -1 */
static int64_t find_edge(const int64_t* ptr, const uint32_t* col, uint32_t u, uint32_t v) {
    int64_t lo = ptr[u], hi = ptr[u + 1];
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (col[mid] < v) lo = mid + 1; else hi = mid;
    }
    return (lo < ptr[u + 1] && col[lo] == v) ? lo : -1;
}

/* ------------------------------------------------------------------ */
/* Algorithm 1: specialized Core Graph.                    */
/* ------------------------------------------------------------------ */

/*
 * Identify (Alg 1 l.13-26): evaluate Q(h) on the given graph; for every edge
 * e(u,v) of that graph with Q(h) having reached u (reading Q6) and
 * Val(u) (+) w(u,v) == Val(v), add e(u,v) (direction f) or e(v,u)
 * (direction b) to E_c.  flags are indexed by G's CSR edge position.
 */
static void identify(int kind, int64_t n, const int64_t* gptr, const uint32_t* gadj,
                     const uint32_t* gwt, int dir_b, const int64_t* Gptr, const uint32_t* Gcol,
                     uint32_t h, uint8_t* flags, uint32_t* val) {
    or_query(kind, n, gptr, gadj, gwt, h, val);                       /* l.14 */
    for (int64_t u = 0; u < n; ++u) {                                 /* l.15 */
        if (!reached(kind, val[u])) continue;                         /* l.16 */
        for (int64_t i = gptr[u]; i < gptr[u + 1]; ++i) {
            uint32_t v = gadj[i];
            uint32_t cand = or_extend(kind, val[u], kind == K_BFS ? 1u : gwt[i]);
            if (cand != val[v]) continue;                             /* l.17 */
            if (!dir_b) flags[i] = 1;                                 /* l.19 */
            else {
                int64_t e = find_edge(Gptr, Gcol, v, (uint32_t)u);    /* l.21: e(v,u) in G */
                if (e >= 0) flags[e] = 1;
            }
        }
    }
}

/* the connectivity edge of Alg 1 l.8-12 for row v: min w (max w for SSWP), ties -> smaller dst */
static int64_t connectivity_edge(int kind, const int64_t* ptr, const uint32_t* wt, int64_t v) {
    int64_t best = ptr[v];
    for (int64_t i = ptr[v] + 1; i < ptr[v + 1]; ++i) {
        if (kind == K_BFS || kind == K_REACH) break;          /* any edge: the first */
        if (kind == K_SSWP ? (wt[i] > wt[best]) : (wt[i] < wt[best])) best = i;
    }
    return best;
}

/*
 * Alg 1 for hubs[0..K): flags (u8[m], G's CSR order) receives E_c.
 * connectivity != 0 applies l.8-12.  Returns |E_c|.
 */
int64_t or_cg_alg1(int kind, int64_t n, const int64_t* ptr, const uint32_t* col, const uint32_t* wt,
                   const int64_t* cptr, const uint32_t* crow, const uint32_t* cwt, int32_t K,
                   const uint32_t* hubs, int connectivity, uint8_t* flags) {
    int64_t m = ptr[n];
    memset(flags, 0, (size_t)m);
    uint32_t* val = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)n);
    for (int32_t k = 0; k < K; ++k) {                                           /* l.3 */
        identify(kind, n, ptr, col, wt, 0, ptr, col, hubs[k], flags, val);      /* l.4 */
        identify(kind, n, cptr, crow, cwt, 1, ptr, col, hubs[k], flags, val);   /* l.5 */
    }
    if (connectivity) {
        for (int64_t v = 0; v < n; ++v) {                                       /* l.8 */
            if (ptr[v + 1] == ptr[v]) continue;                                 /* OutDegree(v) != 0 */
            int any = 0;
            for (int64_t i = ptr[v]; i < ptr[v + 1]; ++i) any |= flags[i];
            if (!any) flags[connectivity_edge(kind, ptr, wt, v)] = 1;           /* l.10 */
        }
    }
    free(val);
    int64_t cnt = 0;
    for (int64_t i = 0; i < m; ++i) cnt += flags[i];
    return cnt;
}

/* ------------------------------------------------------------------ */
/* Algorithm 2: general Core Graph, sequential FIFO.     */
/* ------------------------------------------------------------------ */

/*
 * Traverse (Alg 2 l.10-27) from s with label `lab` over graph (gptr, gadj).
 * dir_b: the graph is G^R; each added edge e(u,v) of G^R is recorded as
 * the G edge e(v,u) (l.9 Reverse).
 */
static void traverse(int64_t n, const int64_t* gptr, const uint32_t* gadj, uint32_t s,
                     uint32_t lab, uint32_t* qid, int dir_b, const int64_t* Gptr,
                     const uint32_t* Gcol, uint8_t* flags, uint32_t* fifo) {
    int64_t head = 0, tail = 0;
    fifo[tail++] = s;                                  /* l.12 (s is not labeled: Q10) */
    while (head < tail) {                              /* l.13 */
        uint32_t u = fifo[head++];                     /* l.14 */
        for (int64_t i = gptr[u]; i < gptr[u + 1]; ++i) {   /* l.15 */
            uint32_t v = gadj[i];
            if (qid[v] != lab) {                       /* l.16 */
                if (!dir_b) flags[i] = 1;              /* l.18 */
                else {
                    int64_t e = find_edge(Gptr, Gcol, v, u);
                    if (e >= 0) flags[e] = 1;
                }
                if (qid[v] == 0) {                     /* l.19 */
                    if (tail >= n + 1) abort();        /* cannot happen: each v labeled once */
                    fifo[tail++] = v;                  /* l.20 */
                    qid[v] = lab;                      /* l.21 */
                }
            }
        }
    }
}

/*
 * Alg 2 for hubs[0..K) (label k+1 for hub k; reading Q10).  per_direction
 * != 0 uses separate Qid arrays for forward and backward traversals
 * (option of reading Q9); connectivity != 0 adds Alg 1 l.8-12 edges
 * (option of reading Q11).  Returns |E_c|.
 */
int64_t or_cg_alg2(int64_t n, const int64_t* ptr, const uint32_t* col, const int64_t* cptr,
                   const uint32_t* crow, int32_t K, const uint32_t* hubs, int per_direction,
                   int connectivity, uint8_t* flags) {
    int64_t m = ptr[n];
    memset(flags, 0, (size_t)m);
    uint32_t* qf = (uint32_t*)calloc((size_t)n, sizeof(uint32_t));           /* l.3 */
    uint32_t* qb = per_direction ? (uint32_t*)calloc((size_t)n, sizeof(uint32_t)) : qf;
    uint32_t* fifo = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(n + 1));
    for (int32_t k = 0; k < K; ++k) {                                         /* l.5 */
        traverse(n, ptr, col, hubs[k], (uint32_t)k + 1u, qf, 0, ptr, col, flags, fifo);   /* l.6 */
        traverse(n, cptr, crow, hubs[k], (uint32_t)k + 1u, qb, 1, ptr, col, flags, fifo); /* l.7 */
    }
    if (connectivity) {
        for (int64_t v = 0; v < n; ++v) {
            if (ptr[v + 1] == ptr[v]) continue;
            int any = 0;
            for (int64_t i = ptr[v]; i < ptr[v + 1]; ++i) any |= flags[i];
            if (!any) flags[ptr[v]] = 1;
        }
    }
    free(fifo);
    if (per_direction) free(qb);
    free(qf);
    int64_t cnt = 0;
    for (int64_t i = 0; i < m; ++i) cnt += flags[i];
    return cnt;
}

/* Sub-graph of G made of the flagged edges (CG(V, E_c)): CSR arrays. */
int64_t or_subgraph(int64_t n, const int64_t* ptr, const uint32_t* col, const uint32_t* wt,
                    const uint8_t* flags, int64_t* sptr, uint32_t* scol, uint32_t* swt) {
    int64_t o = 0;
    sptr[0] = 0;
    for (int64_t u = 0; u < n; ++u) {
        for (int64_t i = ptr[u]; i < ptr[u + 1]; ++i)
            if (flags[i]) { scol[o] = col[i]; swt[o] = wt[i]; ++o; }
        sptr[u + 1] = o;
    }
    return o;
}

/* ------------------------------------------------------------------ */
/* Algorithm 3: 2Phase evaluation, sequential BSP order. */
/* ------------------------------------------------------------------ */

typedef struct {
    int64_t iters_p1, iters_p2, edges_p1, edges_p2, updates_p1, updates_p2;
    int64_t impacted, reached, precise_p1, unvisited_p2;
} or_stats_t;

/*
 * Process (Alg 3 l.21-34): for u in Active (ascending id), for each out-edge
 * e(u,v): if Needed(e) (l.25: the kind's strict "better" test, Table 6),
 * apply EdgeFunction (l.26: sequential CASMIN/CASMAX, which always succeeds
 * when Needed), and add v to newAct when changed or on its first visit in
 * phase 2 (l.27).  Active / newAct are byte maps over V.
 */
static void process(int kind, int64_t n, const int64_t* ptr, const uint32_t* adj,
                    const uint32_t* wt, const uint8_t* act, uint8_t* newact, uint32_t* val,
                    int phase2, uint8_t* visited2, int64_t* edges, int64_t* updates) {
    memset(newact, 0, (size_t)n);
    for (int64_t u = 0; u < n; ++u) {
        if (!act[u]) continue;
        if (phase2) visited2[u] = 1;   /* u pushes its full G out-list in phase 2 */
        for (int64_t i = ptr[u]; i < ptr[u + 1]; ++i) {
            uint32_t v = adj[i];
            uint32_t cand = or_extend(kind, val[u], kind == K_BFS ? 1u : wt[i]);
            ++*edges;
            if (or_better(kind, cand, val[v])) {               /* Needed(e(u,v)) */
                val[v] = cand;                                 /* EdgeFunction */
                ++*updates;
                int change = 1;
                int first = phase2 && !visited2[v];            /* FirstPhase2Visit(v) */
                if (change || first) newact[v] = 1;
            }
        }
    }
}

static int any_set(const uint8_t* a, int64_t n) {
    for (int64_t i = 0; i < n; ++i) if (a[i]) return 1;
    return 0;
}

/* Alg 3 l.3-6 (readings Q2, Q3): returns Active = OutNeighbors_G(s) as a byte map. */
static void init_query(int kind, int64_t n, const int64_t* ptr, const uint32_t* col,
                       const uint32_t* wt, uint32_t s, uint32_t* val, uint8_t* act) {
    const uint32_t INIT = or_init_val(kind);
    for (int64_t v = 0; v < n; ++v) val[v] = INIT;                  /* l.6 */
    memset(act, 0, (size_t)n);
    val[s] = or_source_val(kind);                                   /* l.4 */
    for (int64_t i = ptr[s]; i < ptr[s + 1]; ++i) {                 /* l.5 */
        uint32_t cand = or_extend(kind, val[s], kind == K_BFS ? 1u : wt[i]);
        if (or_better(kind, cand, val[col[i]])) val[col[i]] = cand;
        act[col[i]] = 1;                                            /* l.10 */
    }
}

/*
 * 2Phase (Alg 3): phase 1 on CG (cg_ptr/cg_col/cg_wt) from OutNeighbors_G(s),
 * then phase 2 on G from the impacted set {v : Val(v) != InitVal}
 * (reading Q4), with Reduced(E) = E (main evaluation).
 * p1 (nullable) receives the values after phase 1.
 */
void or_2phase(int kind, int64_t n, const int64_t* ptr, const uint32_t* col, const uint32_t* wt,
               const int64_t* cg_ptr, const uint32_t* cg_col, const uint32_t* cg_wt, uint32_t s,
               uint32_t* val, uint32_t* p1, or_stats_t* st) {
    or_stats_t z;
    memset(&z, 0, sizeof z);
    uint8_t* act = (uint8_t*)malloc((size_t)n);
    uint8_t* nxt = (uint8_t*)malloc((size_t)n);
    uint8_t* visited2 = (uint8_t*)calloc((size_t)n, 1);
    init_query(kind, n, ptr, col, wt, s, val, act);                 /* l.3-8 */
    while (any_set(act, n)) {                                       /* l.11 */
        process(kind, n, cg_ptr, cg_col, cg_wt, act, nxt, val, 0, visited2, &z.edges_p1, &z.updates_p1);
        uint8_t* t = act; act = nxt; nxt = t;                       /* l.12 */
        ++z.iters_p1;
    }
    if (p1) memcpy(p1, val, sizeof(uint32_t) * (size_t)n);
    for (int64_t v = 0; v < n; ++v) {                               /* l.15 */
        act[v] = reached(kind, val[v]) ? 1 : 0;
        z.impacted += act[v];
    }
    while (any_set(act, n)) {                                       /* l.16 */
        process(kind, n, ptr, col, wt, act, nxt, val, 1, visited2, &z.edges_p2, &z.updates_p2);
        uint8_t* t = act; act = nxt; nxt = t;                       /* l.17 */
        ++z.iters_p2;
    }
    for (int64_t v = 0; v < n; ++v) {
        if (v == s || !reached(kind, val[v])) continue;
        ++z.reached;
        if (p1 && p1[v] == val[v]) ++z.precise_p1;
        if (!visited2[v] && ptr[v + 1] > ptr[v]) ++z.unvisited_p2;
    }
    if (st) *st = z;
    free(act);
    free(nxt);
    free(visited2);
}

/* FULL mode (the baseline): Alg 3 init, then Process on G until Active is empty. */
void or_full_bsp(int kind, int64_t n, const int64_t* ptr, const uint32_t* col, const uint32_t* wt,
                 uint32_t s, uint32_t* val, or_stats_t* st) {
    or_stats_t z;
    memset(&z, 0, sizeof z);
    uint8_t* act = (uint8_t*)malloc((size_t)n);
    uint8_t* nxt = (uint8_t*)malloc((size_t)n);
    init_query(kind, n, ptr, col, wt, s, val, act);
    while (any_set(act, n)) {
        process(kind, n, ptr, col, wt, act, nxt, val, 0, NULL, &z.edges_p2, &z.updates_p2);
        uint8_t* t = act; act = nxt; nxt = t;
        ++z.iters_p2;
    }
    for (int64_t v = 0; v < n; ++v)
        if (v != s && reached(kind, val[v])) ++z.reached;
    if (st) *st = z;
    free(act);
    free(nxt);
}

/* ---------------------------------------------------------------- WCC (NEXT-3)
 * Weakly connected components, the fixpoint of Table 6's WCC row: label
 * propagation from Val(v) = v with CASMIN over both edge directions converges to the minimum
 * vertex id of v's weakly connected component.  The oracle computes that definition directly:
 * union-find over the undirected edges, then the smallest id of every set. */
static int64_t uf_find(int64_t* par, int64_t x) {
    while (par[x] != x) {
        par[x] = par[par[x]];
        x = par[x];
    }
    return x;
}

void or_wcc(int64_t n, const int64_t* ptr, const uint32_t* col, uint32_t* out) {
    int64_t* par = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    for (int64_t v = 0; v < n; ++v) par[v] = v;
    for (int64_t u = 0; u < n; ++u)
        for (int64_t e = ptr[u]; e < ptr[u + 1]; ++e) {
            int64_t a = uf_find(par, u), b = uf_find(par, (int64_t)col[e]);
            if (a == b) continue;
            if (a < b) par[b] = a; else par[a] = b; /* the root is the smaller id */
        }
    for (int64_t v = 0; v < n; ++v) out[v] = (uint32_t)uf_find(par, v);
    free(par);
}

/* ---------------------------------------------------------------- O7 (NEXT-1)
 * Which phase-1 values are PROVEN precise.  p1 = Val(s, v) on the CG after phase 1;
 * hf[k*n + v] = Q(h_k) on G at v (forward Identify query, "d(h, v).G"), hb[k*n + v] = Q(h_k) on
 * G^R at v ("d(v, h).G"), for the K hubs the CG was built from.  out[v] = 1 iff v is reached in
 * phase 1 and some hub certifies it:
 *   SSSP / BFS, Theorem 1:
 *     (a) p1(v) == d(s,h) - d(v,h)      (b) p1(v) == d(h,v) - d(h,s)
 *     (the right-hand sides are lower bounds of d(s,v) by the triangle inequality, P:1338-1366;
 *     p1 is an upper bound because CG is a subgraph of G; both d's must be finite)
 *   SSWP (max of path minima; p1 <= W(s,v) because CG is a subgraph): the bottleneck triangle
 *     W(s,h) >= min(W(s,v), W(v,h)) gives, when W(v,h) > W(s,h), the upper bound W(s,v) <= W(s,h);
 *     likewise W(h,v) >= min(W(h,s), W(s,v)) gives W(s,v) <= W(h,v) when W(h,s) > W(h,v).
 *     (a) W(v,h) > W(s,h) and p1(v) == W(s,h)     (b) W(h,s) > W(h,v) and p1(v) == W(h,v)
 *   SSNP (min of path maxima; p1 >= N(s,v)): mirror images,
 *     (a) N(v,h) < N(s,h) and p1(v) == N(s,h)     (b) N(h,s) < N(h,v) and p1(v) == N(h,v)
 *   REACH: p1(v) == 1 (the lattice top, final by definition).
 * Viterbi has no exact certificate here (its triangle bound needs a rounded division). */
void or_certified(int kind, int64_t n, uint32_t s, const uint32_t* p1, int32_t K, const uint32_t* hf,
                  const uint32_t* hb, uint8_t* out) {
    const uint32_t INF = 0xFFFFFFFFu;
    for (int64_t v = 0; v < n; ++v) {
        out[v] = 0;
        const uint32_t p = p1[v];
        if (p == or_init_val(kind)) continue;                        /* not reached in phase 1 */
        if (kind == K_REACH) { out[v] = p == 1u; continue; }
        for (int32_t k = 0; k < K && !out[v]; ++k) {
            const uint32_t* f = hf + (size_t)k * (size_t)n;         /* d(h, .) */
            const uint32_t* b = hb + (size_t)k * (size_t)n;         /* d(., h) */
            const uint32_t d_sh = b[s], d_vh = b[v], d_hv = f[v], d_hs = f[s];
            if (kind == K_SSSP || kind == K_BFS) {
                if (d_sh != INF && d_vh != INF && d_sh >= d_vh && p == d_sh - d_vh) out[v] = 1;   /* (a) */
                if (d_hv != INF && d_hs != INF && d_hv >= d_hs && p == d_hv - d_hs) out[v] = 1;   /* (b) */
            } else if (kind == K_SSWP) {
                if (d_vh > d_sh && p == d_sh) out[v] = 1;                                        /* (a) */
                if (d_hs > d_hv && p == d_hv) out[v] = 1;                                        /* (b) */
            } else if (kind == K_SSNP) {
                if (d_vh < d_sh && p == d_sh) out[v] = 1;                                        /* (a) */
                if (d_hs < d_hv && p == d_hv) out[v] = 1;                                        /* (b) */
            }
        }
    }
}
