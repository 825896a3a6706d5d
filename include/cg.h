/*
 * include/cg.h — C ABI of the B200-native Core Graph hot path.
 *
 * Method: Jiang et al., "Core Graph: Exploiting Edge Centrality to Speedup
 * the Evaluation of Iterative Graph Queries", EuroSys '24.  Citations
 * "P:<line>" refer to lines of the paper text and the section /
 * algorithm / table they sit in.  Readings of ambiguous passages (Q1..Q20)
 * are listed in DESIGN.md.
 *
 * Conventions for every entry point:
 *   - Returns cg_status; CG_OK == 0.  Nothing throws across the ABI.  On
 *     error, cg_last_error() returns a thread-local detail string.
 *   - "device" pointers are CUDA device memory on the graph's device,
 *     "host" pointers are CPU memory (pinned memory is fastest).
 *   - Input pointers are BORROWED: read during the call (or, for
 *     stream-ordered calls, until the stream reaches the call) and never
 *     retained.  Output buffers are caller-allocated.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  cg_query / cg_rmat_generate are stream-ordered and
 *     asynchronous; cg_graph_create and cg_build synchronise `stream`.
 *   - All calls on one cg_graph share its device workspace.  They may be
 *     issued on different streams: each call's stream first waits (an event,
 *     no host sync) for the previous call on that graph, so the calls run in
 *     issue order.  Calls on one graph must come from one host thread at a
 *     time.
 *   - Errors detected on the DEVICE by an asynchronous call (a source id >= n
 *     in a device array, a narrow output format overflow, an internal
 *     iteration bound) are STICKY per graph: the next query call on the graph
 *     (cg_query*, cg_query_host*) returns that error without doing its own
 *     work, and cg_graph_status() synchronises `stream` and returns it.  Either
 *     clears it.  Calls with `stats` synchronise and return their own device
 *     errors directly.
 *   - No PyTorch types appear here; the Python binding passes raw pointers
 *     (torch tensors' data_ptr) and a raw stream handle.
 *   - Internal device memory comes from the allocator installed with
 *     cg_set_allocator (the Python binding installs PyTorch's caching
 *     allocator), else cudaMalloc.
 */
#ifndef CG_H
#define CG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    CG_OK = 0,
    CG_EINVAL = -1,        /* bad argument: null pointer, source >= n, n_src < 0, K <= 0 or K > n, bad enum */
    CG_ENOMEM = -2,        /* device allocation failed */
    CG_ECUDA = -3,         /* a CUDA runtime error (detail in cg_last_error) */
    CG_ENOCG = -4,         /* cg_query(..., CG_MODE_2PHASE) before cg_build for that kind */
    CG_EOVERFLOW = -5,     /* n >= 2^32-1, m >= 2^32, or (n-1)*w_max >= 2^32-1 (SSSP could wrap);
                              a value not representable in the requested narrow output format */
    CG_EUNSUPPORTED = -7,  /* feature not available on this device (e.g. no cooperative launch) */
    CG_EINTERNAL = -8      /* internal invariant violated (e.g. iteration bound exceeded) */
} cg_status;

/* The six query kinds (north_star; Table 6 P:1496-1535 for SSSP/SSWP/SSNP/Viterbi/REACH;
 * BFS = hop count, reading D1).  Value words are u32 for all kinds except
 * VITERBI, whose value is an IEEE binary32 probability stored in the same 32-bit slot. */
typedef enum { CG_SSSP = 0, CG_SSWP = 1, CG_SSNP = 2, CG_VITERBI = 3, CG_BFS = 4, CG_REACH = 5, CG_WCC = 6 } cg_kind;
/* CG_WCC (Table 6 WCC row P:1532-1535): weakly connected
 * components by label propagation — Val(v) starts at v for every vertex, all vertices active,
 * Needed Val(v) > Val(u), EdgeFunction CASMIN(Val(v), Val(u)), over BOTH edge directions; the
 * fixpoint is the minimum vertex id of v's weakly connected component.  It is a whole-graph
 * query: cg_query takes n_src == 1 (src may be NULL) and writes n labels.  2PHASE runs phase 1
 * on the general Core Graph (Alg 2, shared with BFS / REACH) and phase 2 on G from every
 * vertex (reading W2). */

/* Output formats of the value rows (cg_query_fmt / cg_query_host_fmt).  The values are the same;
 * only their encoding differs (a narrower wire format for gathers and host copies):
 *   CG_OUT_U32   row q = n uint32 words (binary32 for VITERBI) — cg_query's format;
 *   CG_OUT_U16   row q = n uint16: a value < 0xFFFF as itself, 0xFFFFFFFF (InitVal of SSSP / SSNP /
 *                BFS, SourceInitVal of SSWP) as 0xFFFF; any other value >= 0xFFFF is a sticky
 *                CG_EOVERFLOW.  SSSP, SSWP, SSNP, BFS, REACH (not VITERBI, not WCC);
 *   CG_OUT_BITS  REACH only: row q = ceil(n/32) uint32 words, bit (v % 32) of word v/32 = Val(v). */
typedef enum { CG_OUT_U32 = 0, CG_OUT_U16 = 1, CG_OUT_BITS = 2 } cg_out_format;

/* CG_MODE_2PHASE: Algorithm 3 — phase 1 on the Core Graph, phase 2 on G
 * from the impacted set.  CG_MODE_FULL: the baseline, the same relaxation on G only. */
typedef enum { CG_MODE_2PHASE = 0, CG_MODE_FULL = 1 } cg_mode;

/* Hub set H of Algorithm 1: the K highest total-degree vertices (P:464-466,
 * P:1669-1677, reading Q7), K uniformly sampled vertices with outdeg > 0 (north_star,
 * reading D2), or caller-given ids. */
typedef enum { CG_HUBS_TOPDEG = 0, CG_HUBS_SAMPLED = 1, CG_HUBS_GIVEN = 2 } cg_hub_policy;

/* Which Core Graph construction: AUTO = Algorithm 1 (specialized) for
 * SSSP/SSWP/SSNP/VITERBI and Algorithm 2 (general) for BFS/REACH
 * (reading Q12).  GENERAL uses one Qid[] for both traversal directions (the
 * literal Alg 2, reading Q9); GENERAL_PERDIR keeps one Qid[] per direction. */
typedef enum { CG_ALG_AUTO = 0, CG_ALG_SPECIALIZED = 1, CG_ALG_GENERAL = 2, CG_ALG_GENERAL_PERDIR = 3 } cg_cg_alg;

typedef struct cg_graph_s* cg_graph; /* opaque: owns G (CSR), G^R (CSC) and the CGs on one device */

/* Per-query counters (SURVEY §5 tracing; Table 5 / Fig 5 analogs; SURVEY §8(b) cg_stats).  Edge and update
 * counts of the asynchronous GPU relaxation are NOT unique (they depend on timing);
 * impacted / reached / precise_p1 ARE unique.  When queries run batched (several sources per
 * pass, the default for n_src >= 2), iterations and frontier sizes are those of the batch's
 * union frontier and edges / updates are the batch's (edge, query) totals split evenly over
 * its queries. */
typedef struct {
    int64_t iters_p1, iters_p2;      /* BSP iterations of phase 1 (CG) and phase 2 (G or FULL) */
    int64_t edges_p1, edges_p2;      /* edges scanned by Process (Alg 3 l.24) */
    int64_t updates_p1, updates_p2;  /* EdgeFunction calls (l.26): CASMIN/CASMAX atomics issued when Needed (Fig 5 ATOMIC) */
    int64_t frontier_p1, frontier_p2;/* sum over iterations of |Active| */
    int64_t impacted;                /* |Active| at the start of phase 2 (Alg 3 l.15, reading Q4) */
    int64_t reached;                 /* |{v != s : Val(v) != InitVal}| after the query */
    int64_t precise_p1;              /* |{v != s reached : p1(v) == final(v)}| (Table 5, reading Q16);
                                        -1 unless the query kept phase-1 values */
    int64_t scanned_p1, scanned_p2;  /* edge words the kernel read (pull sweep: in-edges).  Single-query
                                        engine: == edges_*.  Batched: the union frontier's edges, each
                                        read once for all queries of the batch, split evenly over them */
    int32_t batch_queries;           /* queries per pass of the engine that ran this query (1: single-query) */
    int32_t row_bytes;               /* bytes of one vertex's value row in that pass (u32 lanes: 4 per query;
                                        binary16 lanes: 2 per query; REACH bit lanes: 1 bit per query) */
    float ms_p1;                     /* device time of init + phase 1 (Alg 3 l.3-13) of the pass that ran
                                        this query (0 in FULL mode: everything is phase 2) */
    float ms_p2;                     /* device time of phase 2 (l.14-18) + writing the values out; the
                                        queries of one batched pass share their pass's two times */
} cg_stats;

typedef void* (*cg_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*cg_free_fn)(void* ptr, void* stream, void* ctx);

/* Install the device allocator used for all internal memory (NULL, NULL restores cudaMalloc). */
cg_status cg_set_allocator(cg_alloc_fn alloc, cg_free_fn free_fn, void* ctx);

/*
 * Build G(V,E) on `device` from an edge list of m directed weighted edges
 * (src[i] -> dst[i], weight w[i] >= 1), device pointers, borrowed.
 * Canonicalises (reading Q14): drops self-loops, collapses parallel edges to the minimum
 * weight, sorts rows by destination; builds the CSR of G and the CSC (= CSR of G^R,
 * Alg 1 l.5 P:741, Alg 2 l.7 P:1043).  Vertex ids must be < n.
 * Errors: CG_EINVAL (null pointers with m > 0, n <= 0, an id >= n, a weight 0),
 *         CG_EOVERFLOW (see above), CG_ENOMEM, CG_ECUDA.  Synchronises `stream`.
 */
cg_status cg_graph_create(int device, int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst,
                          const uint32_t* w, void* stream, cg_graph* out);

/* Release every device buffer owned by g (g may be NULL). */
cg_status cg_graph_destroy(cg_graph g);

/* Sizes of the canonical graph: n vertices, m edges, maximum weight.  Any output may be NULL. */
cg_status cg_graph_info(cg_graph g, int64_t* n, int64_t* m, uint32_t* w_max);

/* Copy the canonical CSR (transpose = 0) or CSC (transpose = 1) into caller device buffers:
 * ptr int64[n+1], idx uint32[m] (destinations for CSR, sources for CSC), w uint32[m]; idx and
 * w may both be NULL to copy the row offsets only.  Stream-ordered. */
cg_status cg_graph_export(cg_graph g, int transpose, int64_t* ptr, uint32_t* idx, uint32_t* w, void* stream);

/*
 * Build the Core Graph CG(V, E_c) used by `kind` (Algorithm 1 P:727-786 or Algorithm 2
 * P:1022-1085, see cg_cg_alg), from K hubs chosen by `policy` (`hubs`: host array of K
 * ids, CG_HUBS_GIVEN only; `seed`: CG_HUBS_SAMPLED only).  connectivity != 0 applies
 * Alg 1 l.8-12 (one out-edge for every vertex with outdeg > 0, reading Q8);
 * the default (cg_build) applies it to Algorithm 1 CGs and not to Algorithm 2 CGs
 * (reading Q11).  BFS and REACH share one general CG.  Rebuilding replaces the old CG.
 * Errors: CG_EINVAL (K <= 0, K > n, bad policy / hubs), CG_ENOMEM, CG_ECUDA.
 * Synchronises `stream`.
 */
cg_status cg_build(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs,
                   uint64_t seed, void* stream);
cg_status cg_build_ex(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs,
                      uint64_t seed, cg_cg_alg alg, int32_t connectivity, void* stream);

/*
 * NEXT-4 sharded construction.  Algorithm 1 marks, for every hub, the tight
 * edges of its forward and backward Identify queries and takes the union, so the
 * hubs can be split across GPUs: cg_build_partial marks the flags of hubs [hub_begin, hub_end)
 * of the K hubs `policy` selects (the same K on every rank) into `flags` (device, uint8[m], G's
 * CSR order; zeroed first, no connectivity edges); the caller OR-reduces the ranks' flags
 * (e.g. ncclAllReduce(ncclUint8, ncclMax)); cg_build_from_flags installs the merged flags as
 * the kind's Core Graph, adding the connectivity edges (connectivity < 0: Alg 1's default, on)
 * and compacting.  SSSP / SSWP / SSNP / Viterbi only: Algorithm 2 (BFS / REACH) labels
 * vertices across hubs in order and is not split (CG_EUNSUPPORTED).  Merged
 * builds keep no NEXT-1 hub certificates.  Both synchronise `stream`.
 */
cg_status cg_build_partial(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs,
                           uint64_t seed, int32_t hub_begin, int32_t hub_end, uint8_t* flags, void* stream);
cg_status cg_build_from_flags(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs,
                              uint64_t seed, const uint8_t* flags, int32_t connectivity, void* stream);

/*
 * NEXT-4 persistence: the CG is identified once and used for all future queries.
 * cg_core_save writes the kind's Core Graph (edge flags bit-packed in G's CSR order, hubs,
 * algorithm, connectivity option) to the host file `path`; cg_core_load installs it for `kind`
 * on a graph with the same n, m and canonical-CSR fingerprint (else CG_EINVAL), without the
 * Identify queries.  CG_ENOCG (save before build), CG_EINVAL (I/O error, foreign or truncated
 * file).  Both synchronise `stream`.
 */
cg_status cg_core_save(cg_graph g, cg_kind kind, const char* path, void* stream);
cg_status cg_core_load(cg_graph g, cg_kind kind, const char* path, void* stream);

/* Core Graph sizes for `kind`: m_cg edges, K hubs (hubs: host buffer of >= K entries, may be NULL),
 * build_ms = device time of the last cg_build for that kind.  CG_ENOCG if not built. */
cg_status cg_core_info(cg_graph g, cg_kind kind, int64_t* m_cg, int32_t* K, uint32_t* hubs, float* build_ms);

/* Copy the Core Graph's edge membership as flags (uint8[m], device, 1 = edge in E_c) in G's
 * canonical CSR edge order.  Stream-ordered.  CG_ENOCG if not built. */
cg_status cg_core_export(cg_graph g, cg_kind kind, uint8_t* flags, void* stream);

/*
 * Evaluate n_src vertex queries Q(s) of `kind`, writing Val(*) of query q to
 * out[q*n .. q*n+n) (device, uint32 words; binary32 for VITERBI).  Unreached vertices hold
 * InitVal, out[q*n + s] = SourceInitVal (reading Q1).  src: device array of n_src ids.
 * mode: CG_MODE_2PHASE (Alg 3: init, phase 1 on CG, phase 2 on G from the impacted set) or
 * CG_MODE_FULL.  The results of both modes are identical.
 * p1_out (device, nullable): phase-1 values per query (2PHASE only), enables precise_p1.
 * stats (host, nullable, n_src entries): per-query counters; if non-NULL the call
 * synchronises `stream` and reports this call's device errors; else it is fully asynchronous
 * (no host synchronisation; one persistent kernel launch, plus for SSSP / BFS a second launch
 * that exits at once unless the binary16 value lanes overflowed, reading N3) and device errors
 * are sticky (see the conventions above).
 * Errors: CG_EINVAL (also: n_src > 0 with a NULL src, except CG_WCC), CG_ENOCG, CG_ENOMEM,
 * CG_ECUDA, CG_EINTERNAL, or a pending sticky error of an earlier call.
 */
cg_status cg_query(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, void* out,
                   cg_stats* stats, void* stream);
cg_status cg_query_ex(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, void* out,
                      void* p1_out, cg_stats* stats, void* stream);

/* cg_query_ex with an output format (cg_out_format): out holds n_src rows in that format. */
cg_status cg_query_fmt(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode,
                       cg_out_format fmt, void* out, void* p1_out, cg_stats* stats, void* stream);

/* Synchronise `stream`, then return (and clear) the graph's sticky device error (CG_OK if none):
 * CG_EINVAL for a source id >= n passed in a device array to an asynchronous query (its row holds
 * InitVal), CG_EOVERFLOW for a narrow-format overflow, CG_EINTERNAL for an iteration bound. */
cg_status cg_graph_status(cg_graph g, void* stream);

/*
 * End-to-end variant with HOST buffers: src (host, n_src ids) and out (host, n_src*n words).
 * Copies sources host->device, runs the queries in device batches of `batch` (<= 0: about 512 MiB
 * of result rows, rounded down to whole passes of the batched engine — 32 queries, 16 for u32 lanes)
 * and streams each batch's values device->host on the graph's copy stream while the next batch
 * computes (two device result slots, kept by the graph between calls).  Synchronises `stream`
 * before returning; out is complete and the call's device errors are returned.
 */
cg_status cg_query_host(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, void* out,
                        int32_t batch, void* stream);
/* The same with an output format (cg_out_format): out (host) holds n_src rows in that format. */
cg_status cg_query_host_fmt(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode,
                            cg_out_format fmt, void* out, int32_t batch, void* stream);

/*
 * Asynchronous cg_query_host_fmt: enqueues the source copy, the queries and the result copies and
 * returns without synchronising.  The result copies run on the graph's own copy stream, so they
 * overlap the computation of the next call on the graph (a multi-kind step drains kind k's rows
 * while kind k+1 computes).  out is complete once cg_graph_status(g, stream) returns (it waits for
 * `stream` and the graph's copy stream, and returns the device errors of the calls), or once a
 * later synchronous cg_query_host* call on the graph returns; synchronising `stream` alone is not
 * enough.  out must be pinned host memory for the copies to overlap and stay valid until then;
 * src (any host memory) is staged before the call returns.  Host-checkable errors return at once.
 */
cg_status cg_query_host_async(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode,
                              cg_out_format fmt, void* out, int32_t batch, void* stream);

/*
 * Device twin of the seeded R-MAT input generator (gen/rmat.c defines it): edges
 * [e0, e0+count) into device arrays src/dst/w.  tA/tAB/tABC are the integer quadrant
 * thresholds floor(p*2^32).  Stream-ordered.
 */
cg_status cg_rmat_generate(uint64_t n, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max, uint64_t seed,
                           int32_t permute, uint64_t e0, uint64_t count, uint32_t* src, uint32_t* dst, uint32_t* w,
                           void* stream);

/* Number of CUDA kernels this library has launched in this process (for launch accounting). */
int64_t cg_kernel_launches(void);

/* Human-readable name of a status code, and the thread-local detail of the last error. */
const char* cg_status_string(cg_status s);
const char* cg_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* CG_H */
