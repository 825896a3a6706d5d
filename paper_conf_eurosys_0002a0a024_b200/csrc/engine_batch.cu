// engine_batch.cu — SURVEY §8(f) NEXT-2: batched multi-source relaxation.  B independent
// queries of one kind (vertex queries are independent) run through Alg 3
// in lock-step on one persistent kernel:
//
//   * values live as V[v][q] (a 32·B-byte row per vertex), so ONE gather of v's row serves the
//     Needed test of all B queries: the random-access cost that bounds the single-query sweep
//     (one 32 B sector per edge per query) drops B-fold;
//   * the frontier is the union over the batch: a vertex bitmap plus a per-vertex mask M[v]
//     of the queries for which v is active; phase 1 / phase 2 switch when the union converges;
//   * a lane handles one edge for all B queries: one edge word, one vector load of v's row,
//     u's row from shared memory, B Needed tests, red.min/max only for the needed queries;
//   * the same S1 / S2 structure as engine.cu (CTA-aggregated compaction, edge-balanced split
//     of the union frontier's edges over all warps, red.min / red.max EdgeFunction);
//   * finally the batch is transposed into the caller's [query][vertex] layout.
#include <cstdio>
#include <cstdlib>

#include "kernels.cuh"


namespace cgb {

namespace {

using namespace kern;

constexpr int BT = 512;          // threads per CTA
constexpr int BW = BT / 32;      // warps per CTA

enum { ST_IT1, ST_IT2, ST_E1, ST_E2, ST_U1, ST_U2, ST_F1, ST_F2, ST_IMP, ST_REACH, ST_PREC, ST_S1, ST_S2, NSTAT };
enum { CT0 = 8, CTS = 2, CT_LIST = 0, CT_ACTIVE = 1 };

struct BParams {
    uint32_t n, words, dbits, dmask;
    GraphView G, C;
    const uint32_t* srcs;
    int32_t n_src;
    int two_phase;
    uint32_t* out;              // caller layout: out[q * n + v]
    uint32_t* p1;               // nullable, caller layout
    uint32_t* V;                // [n][B] batch values
    uint32_t* M;                // [n] active-query masks
    uint32_t* bitmap;           // [words] union frontier
    uint32_t* lv;               // compacted union frontier: vertex, edge offset, query mask
    uint32_t* lo;
    uint32_t* lm;
    unsigned long long* ctrl;   // [0] barrier; [CT0 + CTS*slot + k] per-iteration counters
    unsigned long long* stats;  // nullable: per query NSTAT counters
    uint32_t* err;
    uint32_t max_iters;
    uint32_t bits_below;        // frontiers smaller than this keep a bitmap (else the masks M are scanned)
    GraphView R;                // G^R: in-edges for the NEXT-1 pull
    const uint32_t* HB;         // CG hub rows [n][2K] for the certificates (nullable)
    uint32_t K, KP;             // hubs in HB; row stride 2*KP (KP = K rounded up to a multiple of 4)
    int reduced;                // phase 2 starts with the certificate-driven pull (NEXT-1)
    uint32_t fresh;             // bit p-1: phase p pre-reads values from L2 instead of L1
    unsigned long long* trace;  // nullable: per iteration {t_start, t_s1, t_s2, phase<<62|q0<<32|listed, active<<32|edges}
    uint32_t trace_cap;
};

// does row v hold a non-InitVal value for any query (and which)?
template <int KIND, int B>
__device__ __forceinline__ uint32_t row_mask(const uint32_t* V, uint32_t v) {
    using O = Op<KIND>;
    uint32_t m = 0;
    const uint4* r = reinterpret_cast<const uint4*>(V + (size_t)v * B);
#pragma unroll
    for (int i = 0; i < B / 4; ++i) {
        uint4 x;
        asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "l"(r + i));
        m |= (uint32_t)(x.x != O::INIT) << (4 * i) | (uint32_t)(x.y != O::INIT) << (4 * i + 1) |
             (uint32_t)(x.z != O::INIT) << (4 * i + 2) | (uint32_t)(x.w != O::INIT) << (4 * i + 3);
    }
    return m;
}

// ------------------------------------------------------------------ NEXT-1 certificates
// p = Val(s,v) after phase 1 on the CG, a bound on the true value from the "worse" side.
// Fv/Rv = Q(h) on G / on G^R at v, Fs/Rs the same at the source.  A certificate is a bound
// from the other side, met with equality (Theorem 1; bottleneck analogs):
//   SSWP (p <= W(s,v)): W(v,h) > W(s,h) => W(s,v) <= W(s,h);  W(h,s) > W(h,v) => W(s,v) <= W(h,v)
//   SSNP (p >= N(s,v)): N(v,h) < N(s,h) => N(s,v) >= N(s,h);  N(h,s) < N(h,v) => N(s,v) >= N(h,v)
//   SSSP (p >= d(s,v)): d(s,v) >= d(s,h) - d(v,h);  d(s,v) >= d(h,v) - d(h,s)  (Theorem 1), with
//        "infinite minus finite" = infinite (s cannot reach v when v reaches h but s does not, ...)
template <int KIND>
__device__ __forceinline__ bool certified(uint32_t p, uint32_t Fv, uint32_t Rv, uint32_t Fs, uint32_t Rs) {
    if (KIND == CG_SSWP) return (Rv > Rs && p == Rs) || (Fs > Fv && p == Fv);
    if (KIND == CG_SSNP) return (Rv < Rs && p == Rs) || (Fs < Fv && p == Fv);
    if (KIND == CG_SSSP) {
        constexpr uint32_t INF = 0xffffffffu;
        if (Rv != INF && p == (Rs == INF ? INF : (Rs > Rv ? Rs - Rv : 0u))) return true;
        if (Fs != INF && p == (Fv == INF ? INF : (Fv > Fs ? Fv - Fs : 0u))) return true;
    }
    return false;
}

// queries q < nq whose phase-1 value at v is not proven final (Reduced(E) keeps v's in-edges).
// Kept register-light (it runs inside the persistent kernel): the value row is only compared,
// then each open query re-reads its value and scans the hub row 4 hubs per 16 B load.
template <int KIND, int B>
__device__ uint32_t uncertified(const BParams& P, const uint32_t* sh, int nq, uint32_t v) {
    using O = Op<KIND>;
    const uint32_t* row = P.V + (size_t)v * B;
    uint32_t unc = 0;
#pragma unroll
    for (int i = 0; i < B / 4; ++i) {
        uint4 x;
        asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w)
                     : "l"(reinterpret_cast<const uint4*>(row) + i));
        unc |= (uint32_t)(x.x != O::SRC) << (4 * i) | (uint32_t)(x.y != O::SRC) << (4 * i + 1) |
               (uint32_t)(x.z != O::SRC) << (4 * i + 2) | (uint32_t)(x.w != O::SRC) << (4 * i + 3);
    }
    unc &= nq >= 32 ? 0xffffffffu : ((1u << nq) - 1u);  // the lattice top (REACH: reached) is final
    if (KIND == CG_REACH || P.HB == nullptr || !unc) return unc;
    // hub row of v: F at [0, KP), R at [KP, 2 KP) (KP = K rounded up to 4: 16 B aligned chunks)
    const uint32_t K = P.K, KP = P.KP;
    const uint4* hb = reinterpret_cast<const uint4*>(P.HB + (size_t)v * 2 * KP);
    uint32_t todo = unc;
    while (todo) {
        const int q = __ffs(todo) - 1;
        todo &= todo - 1;
        const uint32_t p = ld_cg(row + q);
        const uint32_t* sq = sh + q * 2 * K;
        for (uint32_t h0 = 0; h0 < K; h0 += 4) {
            const uint4 f = __ldg(hb + h0 / 4), r = __ldg(hb + (KP + h0) / 4);
            bool c = false;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const uint32_t h = h0 + j;
                const uint32_t Fv = j == 0 ? f.x : j == 1 ? f.y : j == 2 ? f.z : f.w;
                const uint32_t Rv = j == 0 ? r.x : j == 1 ? r.y : j == 2 ? r.z : r.w;
                c |= h < K && certified<KIND>(p, Fv, Rv, sq[h], sq[K + h]);
            }
            if (c) {
                unc &= ~(1u << q);
                break;
            }
        }
    }
    return unc;
}

// ------------------------------------------------------------------ S1 (union frontier)
// mode: F_BITS (frontier bits set by S2), F_MASKS (frontier = {v : M[v] != 0}), F_IMPACTED
// (Alg 3 l.15: v active for q iff Val(v) != InitVal), F_UNCERT (NEXT-1: v active for its
// uncertified queries; degrees are then in-degrees, g = G^R).
enum { F_BITS = 0, F_MASKS = 1, F_IMPACTED = 2, F_UNCERT = 3 };

template <int KIND, int B>
__device__ void compact_b(const BParams& P, const GraphView& g, int mode, const uint32_t* sh, int nq,
                          unsigned long long* cnt_slot, unsigned long long* act_slot, uint32_t* sm) {
    const bool predicate = mode == F_IMPACTED;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t W = P.words;
    const uint32_t w0 = (uint32_t)(W * blockIdx.x / gridDim.x), w1 = (uint32_t)(W * (blockIdx.x + 1) / gridDim.x);
    const uint32_t lt = (1u << lane) - 1u;

    uint32_t cnt = 0, edges = 0, active = 0;
    for (uint32_t g0 = w0 + warp * 32; g0 < w1; g0 += BW * 32) {
        const uint32_t wi = g0 + lane;
        uint32_t word = 0;
        if (predicate) {  // Alg 3 l.15 for every query of the batch: v active iff some Val(v) != InitVal
            for (uint32_t j = 0; j < 32; ++j) {
                const uint32_t v = (g0 + j) * 32 + lane;
                const bool act = g0 + j < w1 && v < P.n && row_mask<KIND, B>(P.V, v) != 0;
                const uint32_t bits = __ballot_sync(FULL, act);
                if (lane == j) word = bits;
            }
            if (wi < w1 && word) P.bitmap[wi] = word;
        } else if (mode == F_UNCERT) {  // certificates: the uncertified queries' mask parks in M
            for (uint32_t j = 0; j < 32; ++j) {
                const uint32_t v = (g0 + j) * 32 + lane;
                const uint32_t unc = (g0 + j < w1 && v < P.n) ? uncertified<KIND, B>(P, sh, nq, v) : 0u;
                if (unc) P.M[v] = unc;
                const uint32_t bits = __ballot_sync(FULL, unc != 0);
                if (lane == j) word = bits;
            }
            if (wi < w1) P.bitmap[wi] = word;
        } else if (mode == F_MASKS) {  // union frontier = {v : M[v] != 0}: the last S2 set no bitmap bits
#pragma unroll 8
            for (uint32_t j = 0; j < 32; ++j) {
                const uint32_t v = (g0 + j) * 32 + lane;
                const bool act = g0 + j < w1 && v < P.n && ld_cg(P.M + v) != 0u;
                const uint32_t bits = __ballot_sync(FULL, act);
                if (lane == j) word = bits;
            }
            if (wi < w1) P.bitmap[wi] = word;
        } else if (wi < w1) {
            word = ld_cg(P.bitmap + wi);
        }
        active += __popc(word);
        uint32_t nz = __ballot_sync(FULL, word != 0);
        while (nz) {
            int js[CW];
            uint32_t deg[CW];
            word_degrees(g, P.n, g0, nz, lane, js, deg);
#pragma unroll
            for (int k = 0; k < CW; ++k) {
                if (js[k] < 0) break;
                if ((__shfl_sync(FULL, word, js[k]) >> lane) & 1u) {
                    cnt += deg[k] != 0;
                    edges += deg[k];
                }
            }
        }
    }
    for (int o = 16; o > 0; o >>= 1) {
        cnt += __shfl_xor_sync(FULL, cnt, o);
        edges += __shfl_xor_sync(FULL, edges, o);
        active += __shfl_xor_sync(FULL, active, o);
    }
    if (lane == 0) {
        sm[warp] = cnt;
        sm[BW + warp] = edges;
        if (active) atomicAdd(act_slot, (unsigned long long)active);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tc = 0, te = 0;
        for (int i = 0; i < BW; ++i) {
            const uint32_t c = sm[i], e = sm[BW + i];
            sm[i] = tc;
            sm[BW + i] = te;
            tc += c;
            te += e;
        }
        unsigned long long old = 0;
        if (tc) old = atomicAdd(cnt_slot, ((unsigned long long)tc << 32) | te);
        sm[2 * BW] = (uint32_t)(old >> 32);
        sm[2 * BW + 1] = (uint32_t)old;
    }
    __syncthreads();
    uint32_t pos = sm[2 * BW] + sm[warp];
    uint32_t eb = sm[2 * BW + 1] + sm[BW + warp];
    __syncthreads();

    for (uint32_t g0 = w0 + warp * 32; g0 < w1; g0 += BW * 32) {
        const uint32_t wi = g0 + lane;
        const uint32_t word = (wi < w1) ? ld_cg(P.bitmap + wi) : 0u;
        if (word) P.bitmap[wi] = 0u;
        uint32_t nz = __ballot_sync(FULL, word != 0);
        while (nz) {
            int js[CW];
            uint32_t deg[CW];
            word_degrees(g, P.n, g0, nz, lane, js, deg);
#pragma unroll
            for (int k = 0; k < CW; ++k) {
                if (js[k] < 0) break;
                const uint32_t v = (g0 + js[k]) * 32 + lane;
                const bool act = (__shfl_sync(FULL, word, js[k]) >> lane) & 1u;
                const uint32_t d = act ? deg[k] : 0u;
                uint32_t mask = 0;
                if (act) {
                    if (predicate) {
                        mask = row_mask<KIND, B>(P.V, v);
                    } else {
                        mask = ld_cg(P.M + v);
                        P.M[v] = 0u;  // consumed
                    }
                }
                uint32_t incl = d;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(FULL, incl, o);
                    if (lane >= (uint32_t)o) incl += y;
                }
                const uint32_t bal = __ballot_sync(FULL, d != 0);
                if (d) {
                    const uint32_t i = pos + __popc(bal & lt);
                    P.lv[i] = v;
                    P.lo[i] = eb + incl - d;
                    P.lm[i] = mask;
                }
                pos += __popc(bal);
                eb += __shfl_sync(FULL, incl, 31);
            }
        }
    }
}

// ------------------------------------------------------------------ S2 (lane = edge, vector over queries)
// Same edge-balanced split and 32-row windows as engine.cu; a lane handles one edge for all B
// queries: one edge word, one B-value row of v (vector loads), the row of u from shared memory.
template <int B>
struct Row {
    uint32_t x[B];
    // Needed pre-read of all B values: L1-allocating (may be stale, never better), or from L2
    // (fresher: fewer redundant EdgeFunction atomics where values still change a lot)
    __device__ void load(const uint32_t* p, bool fresh) {
#pragma unroll
        for (int i = 0; i < B / 4; ++i) {
            uint4 t;
            if (fresh)
                asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(t.x), "=r"(t.y), "=r"(t.z), "=r"(t.w)
                             : "l"(p + 4 * i));
            else
                asm volatile("ld.global.ca.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(t.x), "=r"(t.y), "=r"(t.z), "=r"(t.w)
                             : "l"(p + 4 * i));
            x[4 * i] = t.x;
            x[4 * i + 1] = t.y;
            x[4 * i + 2] = t.z;
            x[4 * i + 3] = t.w;
        }
    }
    __device__ void load_smem(const uint32_t* p) {
#pragma unroll
        for (int i = 0; i < B / 4; ++i) {
            const uint4 t = reinterpret_cast<const uint4*>(p)[i];
            x[4 * i] = t.x;
            x[4 * i + 1] = t.y;
            x[4 * i + 2] = t.z;
            x[4 * i + 3] = t.w;
        }
    }
};

template <int KIND, bool PACKED, int B>
__device__ void relax_b(const BParams& P, const GraphView& g, uint32_t count, uint32_t E, uint32_t* xs /* 32*B */,
                        bool set_bits, bool fresh, uint32_t& n_edges, uint32_t& n_upd) {
    using O = Op<KIND>;
    constexpr int U = 2;  // edges per lane in flight
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint64_t NW = (uint64_t)gridDim.x * BW;
    const uint32_t e0 = (uint32_t)((uint64_t)E * gw / NW), e1 = (uint32_t)((uint64_t)E * (gw + 1) / NW);
    if (e0 >= e1) return;

    uint32_t lo = 0, hi = count;
    while (hi - lo > 32) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t p = lo + lane * step;
        const bool le = p < hi && ld_cg(P.lo + p) <= e0;
        const uint32_t k = 31 - __clz(__ballot_sync(FULL, le));
        const uint32_t nlo = lo + k * step;
        hi = min(hi, nlo + step);
        lo = nlo;
    }
    {
        const uint32_t p = lo + lane;
        const bool le = p < hi && ld_cg(P.lo + p) <= e0;
        lo += 31 - __clz(__ballot_sync(FULL, le));
    }
    uint32_t i = lo, e = e0;
    for (;;) {
        const uint32_t idx = i + lane;
        uint32_t off = E, base = 0, v = 0, mask = 0;
        if (idx < count) {
            v = ld_cg(P.lv + idx);
            off = ld_cg(P.lo + idx);
            mask = ld_cg(P.lm + idx);
            base = __ldg(g.ptr + v) - off;
        }
        // the window's 32 source rows (all B queries) into shared memory, coalesced
        __syncwarp();
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint32_t f = r * 32 + lane;  // flat index row*B + q
            const uint32_t vr = __shfl_sync(FULL, v, f / B);
            xs[f] = (i + f / B < count) ? ld_cg(P.V + (size_t)vr * B + f % B) : 0u;
        }
        __syncwarp();
        const uint32_t wend = (i + 32 < count) ? ld_cg(P.lo + i + 32) : E;
        const uint32_t ehi = min(e1, wend);
        for (; e < ehi; e += 32 * U) {
            uint32_t k[U], mk[U];
            bool ok[U];
            EdgeWord<PACKED> wd[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t t = e + u * 32 + lane;
                uint32_t kk = 0;
#pragma unroll
                for (uint32_t st = 16; st > 0; st >>= 1)
                    if (__shfl_sync(FULL, off, kk + st) <= t) kk += st;
                k[u] = kk;
                mk[u] = __shfl_sync(FULL, mask, kk);
                const uint32_t a = __shfl_sync(FULL, base, kk) + t;
                ok[u] = t < ehi;
                if (ok[u]) wd[u].load(g, a);
            }
            uint32_t d[U], w[U];
            Row<B> cur[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (ok[u]) {
                    wd[u].decode(P.dbits, P.dmask, d[u], w[u]);
                    cur[u].load(P.V + (size_t)d[u] * B, fresh);
                }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (!ok[u]) continue;
                Row<B> xu;
                xu.load_smem(xs + k[u] * B);
                uint32_t changed = 0;
#pragma unroll
                for (int q = 0; q < B; ++q) {
                    if (!((mk[u] >> q) & 1u)) continue;
                    ++n_edges;
                    const uint32_t cand = O::ext(xu.x[q], w[u]);
                    if (O::better(cand, cur[u].x[q])) {                       // Needed(e(u,v)), query q
                        O::edge_fn(P.V + (size_t)d[u] * B + q, cand);         // EdgeFunction
                        changed |= 1u << q;
                        ++n_upd;
                    }
                }
                if (changed) {
                    red_or(P.M + d[u], changed);                              // v active for those queries
                    if (set_bits) red_or(P.bitmap + (d[u] >> 5), 1u << (d[u] & 31));  // union frontier bit
                }
            }
        }
        if (ehi >= e1) break;
        e = ehi;
        i += 32;
    }
}

// ------------------------------------------------------------------ NEXT-1 pull (Reduced(E))
// The list holds vertices v with uncertified queries (mask) and their IN-edge offsets; a lane
// takes an in-edge (u -> v, w) of the edge-balanced split and, for each uncertified query q
// with Val(u) reached, applies the Table 6 Needed / EdgeFunction to Val(v): all pushes INTO
// uncertified vertices in one sweep, none into certified ones (their in-edges are removed).
template <int KIND, bool PACKED, int B>
__device__ void relax_pull(const BParams& P, uint32_t count, uint32_t E, uint32_t* xs, uint32_t& n_edges,
                           uint32_t& n_upd) {
    using O = Op<KIND>;
    constexpr int U = 2;
    const GraphView& g = P.R;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint64_t NW = (uint64_t)gridDim.x * BW;
    const uint32_t e0 = (uint32_t)((uint64_t)E * gw / NW), e1 = (uint32_t)((uint64_t)E * (gw + 1) / NW);
    if (e0 >= e1) return;
    uint32_t lo = 0, hi = count;
    while (hi - lo > 32) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t p = lo + lane * step;
        const bool le = p < hi && ld_cg(P.lo + p) <= e0;
        const uint32_t k = 31 - __clz(__ballot_sync(FULL, le));
        const uint32_t nlo = lo + k * step;
        hi = min(hi, nlo + step);
        lo = nlo;
    }
    {
        const uint32_t p = lo + lane;
        const bool le = p < hi && ld_cg(P.lo + p) <= e0;
        lo += 31 - __clz(__ballot_sync(FULL, le));
    }
    uint32_t i = lo, e = e0;
    for (;;) {
        const uint32_t idx = i + lane;
        uint32_t off = E, base = 0, v = 0, mask = 0;
        if (idx < count) {
            v = ld_cg(P.lv + idx);
            off = ld_cg(P.lo + idx);
            mask = ld_cg(P.lm + idx);
            base = __ldg(g.ptr + v) - off;
        }
        __syncwarp();
#pragma unroll
        for (int r = 0; r < B; ++r) {  // current rows of the pulling vertices (for the Needed test)
            const uint32_t f = r * 32 + lane;
            const uint32_t vr = __shfl_sync(FULL, v, f / B);
            xs[f] = (i + f / B < count) ? ld_cg(P.V + (size_t)vr * B + f % B) : 0u;
        }
        __syncwarp();
        const uint32_t wend = (i + 32 < count) ? ld_cg(P.lo + i + 32) : E;
        const uint32_t ehi = min(e1, wend);
        for (; e < ehi; e += 32 * U) {
            uint32_t k[U], mk[U], vk[U];
            bool ok[U];
            EdgeWord<PACKED> wd[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t t = e + u * 32 + lane;
                uint32_t kk = 0;
#pragma unroll
                for (uint32_t st = 16; st > 0; st >>= 1)
                    if (__shfl_sync(FULL, off, kk + st) <= t) kk += st;
                k[u] = kk;
                mk[u] = __shfl_sync(FULL, mask, kk);
                vk[u] = __shfl_sync(FULL, v, kk);
                const uint32_t a = __shfl_sync(FULL, base, kk) + t;
                ok[u] = t < ehi;
                if (ok[u]) wd[u].load(g, a);
            }
            uint32_t src[U], w[U];
            Row<B> xu[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (ok[u]) {
                    wd[u].decode(P.dbits, P.dmask, src[u], w[u]);
                    xu[u].load(P.V + (size_t)src[u] * B, false);
                }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (!ok[u]) continue;
                uint32_t changed = 0;
#pragma unroll
                for (int q = 0; q < B; ++q) {
                    if (!((mk[u] >> q) & 1u)) continue;
                    ++n_edges;
                    if (xu[u].x[q] == O::INIT) continue;  // u unreached for q: nothing to pull
                    const uint32_t cand = O::ext(xu[u].x[q], w[u]);
                    if (O::better(cand, xs[k[u] * B + q])) {              // Needed(e(u,v)), query q
                        O::edge_fn(P.V + (size_t)vk[u] * B + q, cand);    // EdgeFunction
                        changed |= 1u << q;
                        ++n_upd;
                    }
                }
                if (changed) red_or(P.M + vk[u], changed);  // v pushes onward for those queries
            }
        }
        if (ehi >= e1) break;
        e = ehi;
        i += 32;
    }
}

// Batch-total count c (per thread) split evenly over the nq queries' counter k: block sum,
// then thread 0 adds total/nq to each (the remainder to the first).
__device__ __forceinline__ void block_add_split(unsigned long long* stats, int q0, int nq, int k, unsigned long long c,
                                                unsigned long long* sm) {
    const unsigned long long t = block_sum<BW, unsigned long long>(c, sm);
    if (threadIdx.x == 0 && t)
        for (int b = 0; b < nq; ++b)
            atomicAdd(stats + (size_t)(q0 + b) * NSTAT + k, t / nq + (b == 0 ? t % nq : 0));
}

// Add a per-thread count to query (tid % B)'s counter k (grid-stride loops over [n][B] keep the
// thread's query fixed because the stride is a multiple of B).
template <int B>
__device__ __forceinline__ void per_query_add(unsigned long long* stats, int q0, int nq, int k, unsigned long long c) {
#pragma unroll
    for (int o = B; o < 32; o <<= 1) c += __shfl_xor_sync(FULL, c, o);
    const uint32_t lane = threadIdx.x & 31;
    if (lane < (uint32_t)B && (int)lane < nq && c) atomicAdd(stats + (size_t)(q0 + lane) * NSTAT + k, c);
}

// V[v][q] -> dst[(q0+q)*n + v] for q < nq, 32 vertices per warp through shared memory
template <int B>
__device__ void transpose_out(const BParams& P, uint32_t* dst, int q0, int nq, uint32_t* xs) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint32_t NW = gridDim.x * BW;
    for (uint32_t v0 = gw * 32; v0 < P.n; v0 += NW * 32) {
        __syncwarp();
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint32_t f = r * 32 + lane;
            const uint32_t v = v0 + f / B;
            xs[(f / B) * (B + 1) + f % B] = v < P.n ? ld_cg(P.V + (size_t)v * B + f % B) : 0u;
        }
        __syncwarp();
        const uint32_t v = v0 + lane;
        if (v < P.n)
            for (int q = 0; q < nq; ++q) dst[(size_t)(q0 + q) * P.n + v] = xs[lane * (B + 1) + q];
    }
}

template <int KIND, bool PACKED, int B>
__global__ void __launch_bounds__(BT, 1) batch_kernel(BParams P) {
    using O = Op<KIND>;
    __shared__ uint32_t sm_cnt[2 * BW + 2];
    __shared__ unsigned long long sm_red[BW];
    extern __shared__ uint32_t dsm[];  // per warp: 32*(B+1) words; then B*2K source hub values
    uint32_t* xs = dsm + (threadIdx.x >> 5) * 32 * (B + 1);
    uint32_t* sh = dsm + BW * 32 * (B + 1);
    unsigned long long epoch = 0;
    const uint64_t tid = blockIdx.x * (uint64_t)BT + threadIdx.x;
    const uint64_t nthreads = (uint64_t)gridDim.x * BT;
    uint32_t ring = 0;

    for (int q0 = 0; q0 < P.n_src; q0 += B) {
        const int nq = min(B, P.n_src - q0);
        // Alg 3 l.4, l.6 for every query of the batch; masks cleared
        for (uint64_t i = tid; i < (uint64_t)P.n * B; i += nthreads) P.V[i] = O::INIT;
        for (uint64_t v = tid; v < P.n; v += nthreads) P.M[v] = 0u;
        grid_sync(P.ctrl, epoch);
        for (int b = 0; b < nq; ++b) {
            const uint32_t s = __ldg(P.srcs + q0 + b);
            if (s >= P.n) {
                if (tid == 0) atomicOr(P.err, 2u);
                continue;
            }
            if (tid == 0) P.V[(size_t)s * B + b] = O::SRC;
            // l.5, l.10: out-neighbours of s in G
            const uint32_t r0 = __ldg(P.G.ptr + s), r1 = __ldg(P.G.ptr + s + 1);
            for (uint64_t e = r0 + tid; e < r1; e += nthreads) {
                EdgeWord<PACKED> wd;
                wd.load(P.G, (uint32_t)e);
                uint32_t d, w;
                wd.decode(P.dbits, P.dmask, d, w);
                P.V[(size_t)d * B + b] = O::ext(O::SRC, w);
                red_or(P.M + d, 1u << b);
                red_or(P.bitmap + (d >> 5), 1u << (d & 31));
            }
        }
        if (P.HB) {  // the sources' hub values (certificates), per block
            for (uint32_t i = threadIdx.x; i < (uint32_t)nq * 2 * P.K; i += BT) {
                const uint32_t b = i / (2 * P.K), k = i % (2 * P.K);
                const uint32_t s = __ldg(P.srcs + q0 + b);
                const uint32_t col = k < P.K ? k : P.KP + (k - P.K);
                sh[i] = s < P.n ? __ldg(P.HB + (size_t)s * 2 * P.KP + col) : 0u;
            }
        }
        grid_sync(P.ctrl, epoch);

        int phase = P.two_phase ? 1 : 2;
        bool predicate = false;
        bool bits = true;  // the current frontier is in the bitmap (seeds set bits), else in M
        bool pull = false; // this iteration is the NEXT-1 pull over uncertified vertices
        uint32_t iters = 0, n_edges = 0, n_upd = 0;  // (edge, query) pairs of the whole batch
        unsigned long long n_scan = 0;                // union edges read (every thread keeps the sum)
        for (;;) {
            const GraphView& g = (phase == 1) ? P.C : P.G;
            const int slot = ring & 3;
            unsigned long long* ctr = P.ctrl + CT0 + CTS * slot;
            if (tid == 0) {
                unsigned long long* z = P.ctrl + CT0 + CTS * ((ring + 2) & 3);
                z[0] = z[1] = 0ull;
            }
            const unsigned long long t_s0 = (P.trace && tid == 0) ? global_ns() : 0ull;
            const int mode = pull ? F_UNCERT : predicate ? F_IMPACTED : bits ? F_BITS : F_MASKS;
            compact_b<KIND, B>(P, pull ? P.R : g, mode, sh, nq, ctr + CT_LIST, ctr + CT_ACTIVE, sm_cnt);
            grid_sync(P.ctrl, epoch);
            ++ring;
            const unsigned long long ce = ld_cg64(ctr + CT_LIST);
            const uint32_t count = (uint32_t)(ce >> 32), E = (uint32_t)ce;
            const uint32_t tr = ring - 1;
            if (P.trace && tid == 0 && tr < P.trace_cap) {
                unsigned long long* t = P.trace + 5ull * tr;
                t[0] = t_s0;
                t[1] = global_ns();
                t[2] = 0;
                t[3] = ((unsigned long long)phase << 62) | ((unsigned long long)q0 << 32) | count;
                t[4] = (ld_cg64(ctr + CT_ACTIVE) << 32) | E;
            }
            if (P.stats && tid == 0) {
                const unsigned long long a = ld_cg64(ctr + CT_ACTIVE);
                for (int b = 0; b < nq; ++b)  // union frontier, reported for every query of the batch
                    atomicAdd(P.stats + (size_t)(q0 + b) * NSTAT + (phase == 1 ? ST_F1 : ST_F2), a);
            }
            if (E == 0 && pull) {  // nothing uncertified has an in-edge: phase 2 is already final
                pull = false;
                bits = false;
            }
            n_scan += E;
            if (E == 0) {
                if (P.stats && tid == 0 && n_scan)
                    for (int b = 0; b < nq; ++b)
                        atomicAdd(P.stats + (size_t)(q0 + b) * NSTAT + (phase == 1 ? ST_S1 : ST_S2),
                                  n_scan / nq + (b == 0 ? n_scan % nq : 0));
                n_scan = 0;
                if (P.stats) {  // batch totals, attributed evenly to the batch's queries
                    block_add_split(P.stats, q0, nq, phase == 1 ? ST_E1 : ST_E2, n_edges, sm_red);
                    block_add_split(P.stats, q0, nq, phase == 1 ? ST_U1 : ST_U2, n_upd, sm_red);
                    if (tid < (uint64_t)nq)
                        atomicAdd(P.stats + (size_t)(q0 + tid) * NSTAT + (phase == 1 ? ST_IT1 : ST_IT2),
                                  (unsigned long long)iters);
                }
                n_edges = n_upd = 0;
                iters = 0;
                if (phase == 1) {
                    if (P.p1) transpose_out<B>(P, P.p1, q0, nq, xs);
                    if (P.stats) {  // impacted per query (Alg 3 l.15); stride is a multiple of B: q fixed
                        unsigned long long c = 0;
                        for (uint64_t i = tid; i < (uint64_t)P.n * B; i += nthreads) c += ld_cg(P.V + i) != O::INIT;
                        per_query_add<B>(P.stats, q0, nq, ST_IMP, c);
                    }
                    phase = 2;
                    if (P.reduced) pull = true;   // Reduced(E): pull into uncertified vertices
                    else predicate = true;        // Active <- impacted vertices (l.15)
                    continue;
                }
                break;
            }
            if (pull) {  // NEXT-1: one pull sweep, then push from the vertices it changed (masks in M)
                relax_pull<KIND, PACKED, B>(P, count, E, xs, n_edges, n_upd);
                pull = false;
                bits = false;
                grid_sync(P.ctrl, epoch);
                if (P.trace && tid == 0 && tr < P.trace_cap) P.trace[5ull * tr + 2] = global_ns();
                ++iters;
                continue;
            }
            // small frontier: its S2 sets frontier bits (few reds) and the next S1 reads the bitmap;
            // large frontier: no bitmap reds (they contend in L2), the next S1 scans M instead
            bits = count < P.bits_below;
            relax_b<KIND, PACKED, B>(P, g, count, E, xs, bits, (P.fresh >> (phase - 1)) & 1u, n_edges, n_upd);
            predicate = false;
            grid_sync(P.ctrl, epoch);
            if (P.trace && tid == 0 && tr < P.trace_cap) P.trace[5ull * tr + 2] = global_ns();
            if (++iters > P.max_iters) {
                if (tid == 0) atomicOr(P.err, 1u);
                return;
            }
        }
        transpose_out<B>(P, P.out, q0, nq, xs);
        if (P.stats) {  // reached / precise per query (thread's query b = tid % B is fixed)
            const uint32_t b = (uint32_t)(tid % B);
            const uint32_t sb = (int)b < nq ? __ldg(P.srcs + q0 + b) : 0xffffffffu;
            unsigned long long r = 0, pr = 0;
            for (uint64_t i = tid; i < (uint64_t)P.n * B; i += nthreads) {
                const uint32_t v = (uint32_t)(i / B);
                const uint32_t fv = ld_cg(P.V + i);
                if ((int)b < nq && v != sb && fv != O::INIT) {
                    ++r;
                    if (P.p1 && ld_cg(P.p1 + (size_t)(q0 + b) * P.n + v) == fv) ++pr;
                }
            }
            per_query_add<B>(P.stats, q0, nq, ST_REACH, r);
            per_query_add<B>(P.stats, q0, nq, ST_PREC, pr);
        }
        grid_sync(P.ctrl, epoch);  // V / M / bitmap are reused by the next batch
    }
}

template <int KIND, bool PACKED, int B>
void launch_b(const BParams& P, int sms, cudaStream_t s) {
    const size_t smem = ((size_t)BW * 32 * (B + 1) + (size_t)B * 2 * 64) * sizeof(uint32_t);
    static int bps = 0;
    if (!bps) {
        if (smem > 48 * 1024)
            CGB_CUDA(cudaFuncSetAttribute(batch_kernel<KIND, PACKED, B>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)smem));
        CGB_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, batch_kernel<KIND, PACKED, B>, BT, smem));
        CGB_CHECK(bps > 0, CG_EUNSUPPORTED, "batch kernel cannot be resident");
    }
    void* args[] = {(void*)&P};
    CGB_CUDA(cudaLaunchCooperativeKernel((const void*)batch_kernel<KIND, PACKED, B>, dim3(bps * sms), dim3(BT), args,
                                         smem, s));
    count_launch();
}

template <bool PACKED, int B>
void launch_kind_b(int kind, const BParams& P, int sms, cudaStream_t s) {
    switch (kind) {
    case CG_SSSP: launch_b<CG_SSSP, PACKED, B>(P, sms, s); break;
    case CG_SSWP: launch_b<CG_SSWP, PACKED, B>(P, sms, s); break;
    case CG_SSNP: launch_b<CG_SSNP, PACKED, B>(P, sms, s); break;
    case CG_VITERBI: launch_b<CG_VITERBI, PACKED, B>(P, sms, s); break;
    case CG_BFS: launch_b<CG_BFS, PACKED, B>(P, sms, s); break;
    case CG_REACH: launch_b<CG_REACH, PACKED, B>(P, sms, s); break;
    default: throw Error(CG_EINVAL, "bad kind");
    }
}

}  // namespace

int batch_width() {
    const char* e = getenv("CG_BATCH");
    const int b = e ? atoi(e) : 16;
    return (b == 8 || b == 16 || b == 32) ? b : 0;  // 0 (or anything else): single-query engine
}

void run_queries_batched(Graph& G, const QueryCall& c, int B, cudaStream_t s, std::vector<cg_stats>* stats) {
    BatchSpace& w = G.bs;
    const uint32_t words = (G.n + 31) / 32;
    if (w.n != G.n || w.B != (uint32_t)B) {
        w.V.alloc((size_t)G.n * B, s);
        w.M.alloc(G.n ? G.n : 1, s);
        w.bitmap.alloc(words ? words : 1, s);
        w.lv.alloc(G.n ? G.n : 1, s);
        w.lo.alloc(G.n ? G.n : 1, s);
        w.lm.alloc(G.n ? G.n : 1, s);
        w.ctrl.alloc(CT0 + CTS * 4, s);
        w.err.alloc(1, s);
        w.n = G.n;
        w.B = (uint32_t)B;
    }
    DevBuf<unsigned long long> st;
    if (stats) st.alloc((size_t)c.n_src * NSTAT, s);
    BParams P{};
    P.n = G.n;
    P.words = words;
    P.dbits = G.dbits;
    P.dmask = G.dbits >= 32 ? 0xffffffffu : ((1u << G.dbits) - 1u);
    P.G = view(*c.full_adj);
    P.C = c.two_phase ? view(*c.core_adj) : P.G;
    P.R = view(G.gr);
    {   // NEXT-1 (Reduced(E) pull) after phase 1 for the kinds with a certificate; CG_REDUCED is a
        // bitmask over cg_kind.  Default REACH only: its certificate (reached = final) leaves only
        // unreachable vertices; the SSWP / SSNP / SSSP certificates are exact but, united over a
        // 16-query batch, leave ~99 % of the vertices uncertified for some query (measured, C2).
        const char* e = getenv("CG_REDUCED");
        const unsigned mask = e ? (unsigned)strtoul(e, nullptr, 0) : (1u << CG_REACH);
        const Core& core = G.core[core_slot(c.kind)];
        const bool has_cert = c.kind == CG_REACH || (core.hub_k > 0 && core.hub_k <= 64 && core.hub_vals.get());
        P.reduced = c.two_phase && c.core_adj == &core.adj && ((mask >> c.kind) & 1u) && has_cert;
        if (P.reduced && c.kind != CG_REACH) {
            P.HB = core.hub_vals.get();
            P.K = core.hub_k;
            P.KP = (core.hub_k + 3) & ~3u;
        }
    }
    P.srcs = c.srcs;
    P.n_src = c.n_src;
    P.two_phase = c.two_phase;
    P.out = c.out;
    P.p1 = c.two_phase ? c.p1 : nullptr;
    P.V = w.V.get();
    P.M = w.M.get();
    P.bitmap = w.bitmap.get();
    P.lv = w.lv.get();
    P.lo = w.lo.get();
    P.lm = w.lm.get();
    P.ctrl = w.ctrl.get();
    P.stats = stats ? st.get() : nullptr;
    P.err = w.err.get();
    P.max_iters = G.n + 8;
    {
        const char* e = getenv("CG_BITS_BELOW");
        P.bits_below = e ? (uint32_t)strtoul(e, nullptr, 10) : G.n / 256;
        const char* f = getenv("CG_FRESH");
        P.fresh = f ? (uint32_t)strtoul(f, nullptr, 10) : 0u;
    }
    CGB_CUDA(cudaMemsetAsync(w.bitmap.get(), 0, w.bitmap.bytes(), s));
    CGB_CUDA(cudaMemsetAsync(w.ctrl.get(), 0, w.ctrl.bytes(), s));
    CGB_CUDA(cudaMemsetAsync(w.err.get(), 0, 4, s));
    if (stats) CGB_CUDA(cudaMemsetAsync(st.get(), 0, st.bytes(), s));
    static const bool tracing = getenv("CG_TRACE") != nullptr;
    DevBuf<unsigned long long> trace;
    if (tracing) {
        P.trace_cap = 1u << 16;
        trace.alloc(5ull * P.trace_cap, s);
        CGB_CUDA(cudaMemsetAsync(trace.get(), 0, trace.bytes(), s));
        P.trace = trace.get();
    }
    if (G.packed) {
        if (B == 8) launch_kind_b<true, 8>(c.kind, P, G.num_sms, s);
        else if (B == 16) launch_kind_b<true, 16>(c.kind, P, G.num_sms, s);
        else launch_kind_b<true, 32>(c.kind, P, G.num_sms, s);
    } else {
        if (B == 8) launch_kind_b<false, 8>(c.kind, P, G.num_sms, s);
        else if (B == 16) launch_kind_b<false, 16>(c.kind, P, G.num_sms, s);
        else launch_kind_b<false, 32>(c.kind, P, G.num_sms, s);
    }
    if (tracing) {
        std::vector<unsigned long long> h(5ull * P.trace_cap);
        CGB_CUDA(cudaMemcpyAsync(h.data(), trace.get(), trace.bytes(), cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaStreamSynchronize(s));
        unsigned long long t0 = 0;
        for (uint32_t i = 0; i < P.trace_cap && h[5 * i]; ++i) {
            const unsigned long long* t = h.data() + 5 * i;
            if (!t0) t0 = t[0];
            fprintf(stderr, "CG_TRACE kind=%d B=%d it=%u q0=%llu phase=%llu list=%llu active=%llu edges=%llu "
                    "t=%.1f s1=%.1f s2=%.1f us\n", c.kind, B, i, (t[3] >> 32) & 0x3fffffffull, t[3] >> 62,
                    t[3] & 0xffffffffull, t[4] >> 32, t[4] & 0xffffffffull, (t[0] - t0) / 1e3, (t[1] - t[0]) / 1e3,
                    t[2] ? (t[2] - t[1]) / 1e3 : 0.0);
        }
    }
    if (stats) {
        std::vector<unsigned long long> h((size_t)c.n_src * NSTAT);
        uint32_t err = 0;
        CGB_CUDA(cudaMemcpyAsync(h.data(), st.get(), st.bytes(), cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaMemcpyAsync(&err, w.err.get(), 4, cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaStreamSynchronize(s));
        CGB_CHECK(!(err & 2u), CG_EINVAL, "source id >= n");
        CGB_CHECK(!(err & 1u), CG_EINTERNAL, "iteration bound exceeded");
        stats->resize(c.n_src);
        for (int qq = 0; qq < c.n_src; ++qq) {
            const unsigned long long* x = h.data() + (size_t)qq * NSTAT;
            cg_stats& o = (*stats)[qq];
            o.iters_p1 = (int64_t)x[ST_IT1];
            o.iters_p2 = (int64_t)x[ST_IT2];
            o.edges_p1 = (int64_t)x[ST_E1];
            o.edges_p2 = (int64_t)x[ST_E2];
            o.updates_p1 = (int64_t)x[ST_U1];
            o.updates_p2 = (int64_t)x[ST_U2];
            o.frontier_p1 = (int64_t)x[ST_F1];
            o.frontier_p2 = (int64_t)x[ST_F2];
            o.impacted = (int64_t)x[ST_IMP];
            o.reached = (int64_t)x[ST_REACH];
            o.precise_p1 = P.p1 ? (int64_t)x[ST_PREC] : -1;
            o.scanned_p1 = (int64_t)x[ST_S1];
            o.scanned_p2 = (int64_t)x[ST_S2];
        }
    }
}

}  // namespace cgb
