// graph.hpp — device-resident graph store (G, G^R, Core Graphs) and query workspace.
#pragma once

#include <vector>

#include "common.cuh"

namespace cgb {

// Edge arrays are over-allocated by this many bytes so that vectorised / bulk edge reads may
// run past the last edge without leaving the allocation.
constexpr size_t kAdjPadBytes = 4096;
inline size_t adj_alloc_elems(size_t m, size_t elem_bytes) { return m + kAdjPadBytes / elem_bytes; }

// Out-edge structure in the engine's HBM layout:
//   ptr   u32[n+1]  row offsets (m < 2^32 is required)
//   adj   u32[m]    packed edge word dst | (w-1) << dbits      (when w_max-1 fits the high bits)
//   adjw  uint2[m]  (dst, w) pairs                              (otherwise)
struct Adj {
    uint32_t n = 0, m = 0;
    DevBuf<uint32_t> ptr;
    DevBuf<uint32_t> adj;
    DevBuf<uint2> adjw;
};

// What a kernel sees of an out-edge structure: row v = edges [ptr[v], end[v]) of adj / adjw,
// with end == nullptr meaning end[v] = ptr[v+1] (a plain CSR).  The split layout of a Core
// Graph (below) gives phase 1 the rows [ptr[v], cg_end[v]) and phase 2's first sweep the rows
// [cg_end[v], ptr[v+1]) of ONE edge array.
struct GraphView {
    const uint32_t* ptr;
    const uint32_t* end;
    const uint32_t* adj;
    const uint2* adjw;
};

inline GraphView view(const Adj& a) { return GraphView{a.ptr.get(), nullptr, a.adj.get(), a.adjw.get()}; }

// A Core Graph in the split-CSR layout ("the edge lists can
// be organized to separate critical and non-critical edges so that latter can be easily skipped
// during the first phase"): ONE copy of G's edges per Core Graph, each row reordered so that
// its CG edges (canonical order) come first and the others (canonical order) follow:
//   sadj / sadjw   the reordered edges, row v at G's own offsets [ptr[v], ptr[v+1])
//   cg_end u32[n]  end of row v's CG part: CG(V, E_c) = rows [ptr[v], cg_end[v])
// Phase 1 reads the CG rows, phase 2's first sweep the non-CG rows [cg_end[v], ptr[v+1])
// (reading N7), later phase-2 iterations whole rows.  E_c membership in G's canonical edge
// order is kept as a bitmap (cg_core_export, persistence, WCC).
struct Core {
    bool built = false;
    int alg = 0;           // 1 = Algorithm 1 (specialized), 2 = Algorithm 2 (general)
    int connectivity = 0;
    uint32_t m_cg = 0;     // |E_c|
    DevBuf<uint32_t> sadj; // split rows, packed edge words
    DevBuf<uint2> sadjw;   // split rows, (dst, w) pairs (wide layout)
    DevBuf<uint32_t> cg_end;
    DevBuf<uint32_t> fbits;  // E_c membership bits in G's CSR edge order (bit e of word e/32)
    std::vector<uint32_t> hubs;
    float build_ms = 0.f;
    // NEXT-1 certificates (Theorem 1 P:1321-1371 and its bottleneck analogs): the Identify
    // queries' values kept as rows hub_vals[v][0..2K) = (Q(h_k) on G at v | Q(h_k) on G^R at v)
    DevBuf<uint32_t> hub_vals;
    uint32_t hub_k = 0;
    Adj sym;               // WCC: CG ∪ CG^R (built on the first WCC 2Phase query)
    bool sym_built = false;
    // CG^R for the pull of dense phase-1 iterations (engine_batch.cu relax_pull_all): the CSR of
    // the reversed Core Graph, and the vertices with CG in-edges (vertex order) with their first
    // in-edge — a static edge-offset list for the edge-balanced split
    Adj rcg;
    DevBuf<uint32_t> pl_v, pl_lo;
    uint32_t pl_count = 0;
    bool rcg_built = false;
};

struct Workspace {
    uint32_t n = 0;
    DevBuf<uint32_t> bitmap;                // ceil(n/32) frontier bits
    DevBuf<uint32_t> lv;                    // n compacted frontier ids
    DevBuf<uint32_t> lo;                    // n exclusive edge offsets of the frontier rows
    DevBuf<unsigned long long> ctrl;        // grid barrier + per-iteration counters
    DevBuf<unsigned long long> stats;       // per-query counters
    DevBuf<uint32_t> err;                   // error flag
    uint32_t stats_cap = 0;
};

struct BatchSpace {         // engine_batch.cu workspace (one batch of queries per pass)
    uint32_t n = 0, B = 0;
    DevBuf<uint32_t> V;         // [n][row words] value rows
    DevBuf<uint32_t> M;         // [n] active-query masks
    DevBuf<uint32_t> bitmap;    // union frontier
    DevBuf<uint32_t> lv, lo, lm;
    DevBuf<unsigned long long> ctrl;
    DevBuf<uint32_t> err;
    uint32_t* err_h = nullptr;  // pinned host copy of err
    uint32_t* err_host() {
        if (!err_h) CGB_CUDA(cudaMallocHost(&err_h, sizeof(uint32_t)));
        *err_h = 0;
        return err_h;
    }
    BatchSpace() = default;
    BatchSpace(const BatchSpace&) = delete;
    BatchSpace& operator=(const BatchSpace&) = delete;
    ~BatchSpace() {
        if (err_h) cudaFreeHost(err_h);
    }
};

struct HostPath {  // cg_query_host*: persistent result slots, source buffer and copy stream
    DevBuf<uint8_t> slot[2];  // two device result slots: batch b computes into b % 2 while b - 1 drains
    DevBuf<uint32_t> dsrc;    // the call's sources on the device
    cudaStream_t cp = nullptr;                      // device -> host copies
    cudaEvent_t done[2] = {nullptr, nullptr};       // slot k computed (on the call's stream)
    cudaEvent_t drained[2] = {nullptr, nullptr};    // slot k copied out (on cp)
    bool pending[2] = {false, false};               // drained[k] recorded: slot k may still be read
    int next = 0;                                   // slot of the next batch (across calls)
    uint32_t* hsrc[2] = {nullptr, nullptr};         // pinned staging of the sources (any host src works)
    size_t hsrc_n[2] = {0, 0};
    cudaEvent_t src_copied[2] = {nullptr, nullptr}; // each staging buffer's last host -> device copy
    bool src_pending[2] = {false, false};
    int src_next = 0;
    HostPath() = default;
    HostPath(const HostPath&) = delete;
    HostPath& operator=(const HostPath&) = delete;
    ~HostPath() {
        if (cp) cudaStreamSynchronize(cp);
        for (int i = 0; i < 2; ++i) {
            if (src_pending[i]) cudaEventSynchronize(src_copied[i]);
            if (hsrc[i]) cudaFreeHost(hsrc[i]);
            if (src_copied[i]) cudaEventDestroy(src_copied[i]);
        }
        for (int i = 0; i < 2; ++i) {
            if (done[i]) cudaEventDestroy(done[i]);
            if (drained[i]) cudaEventDestroy(drained[i]);
        }
        if (cp) cudaStreamDestroy(cp);
    }
};

struct Graph {
    int device = 0;
    uint32_t n = 0, m = 0, w_max = 0;
    uint32_t dbits = 0;    // bits of the destination id in a packed edge word
    bool packed = false;
    int num_sms = 0;
    Adj g;                 // CSR of G
    Adj gr;                // CSR of G^R (= CSC of G)
    DevBuf<uint32_t> reid; // CSC position -> CSR edge index
    Core core[6];          // indexed by cg_kind (BFS and WCC use the REACH slot: one general CG)
    Adj gsym;              // WCC: G ∪ G^R (built on the first WCC query)
    bool gsym_built = false;
    Workspace ws;
    BatchSpace bs;
    HostPath hp;
    // sticky error word of asynchronous calls (ERR_* bits of the engines), in host-mapped pinned
    // memory: kernels write it through sticky_d, the next API call / cg_graph_status reads sticky_h
    uint32_t* sticky_h = nullptr;
    uint32_t* sticky_d = nullptr;
    // calls on one graph share its workspace: each call's stream waits for the previous call's
    // work on another stream (event `last`), so calls are serialised per graph across streams
    cudaEvent_t last = nullptr;
    cudaStream_t last_stream = nullptr;
    bool last_valid = false;
    Graph() = default;
    Graph(const Graph&) = delete;
    Graph& operator=(const Graph&) = delete;
    ~Graph() {
        if (sticky_h) cudaFreeHost(sticky_h);
        if (last) cudaEventDestroy(last);
    }
};

// engine error bits (both engines); ERR_SOURCE / ERR_ITERS / ERR_NARROW are sticky per graph
enum : uint32_t { ERR_ITERS = 1u, ERR_SOURCE = 2u, ERR_LANE_OVERFLOW = 4u, ERR_NARROW = 8u };

inline int core_slot(int kind) { return (kind == CG_BFS || kind == CG_WCC) ? CG_REACH : kind; }

// views of a built Core Graph C of G (split layout)
inline GraphView core_view(const Graph& G, const Core& C) {   // CG(V, E_c): phase 1
    return GraphView{G.g.ptr.get(), C.cg_end.get(), C.sadj.get(), C.sadjw.get()};
}
inline GraphView rest_view(const Graph& G, const Core& C) {   // G minus E_c: phase 2's first sweep
    return GraphView{C.cg_end.get(), G.g.ptr.get() + 1, C.sadj.get(), C.sadjw.get()};
}
inline GraphView split_view(const Graph& G, const Core& C) {  // G with split rows: phase 2
    return GraphView{G.g.ptr.get(), nullptr, C.sadj.get(), C.sadjw.get()};
}

// graph_build.cu
void build_graph(Graph& G, int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                 cudaStream_t s);
void export_adj(const Graph& G, const Adj& a, int64_t* ptr, uint32_t* idx, uint32_t* w, cudaStream_t s);

// engine.cu
struct QueryCall {
    int kind;
    GraphView full;        // G (or G^R for backward Identify queries); in 2Phase the split rows
    GraphView core;        // CG (phase 1); ignored when two_phase == 0
    GraphView rest;        // G minus the CG (phase 2's first sweep, reading N7); ptr null: use full
    const Core* cg;        // the kind's Core Graph when `core` is it (NEXT-1 certificates), else null
    int two_phase;
    const uint32_t* srcs;  // device
    int32_t n_src;
    void* out;             // n_src rows in out_fmt
    uint32_t* p1;          // nullable (u32 rows)
    bool want_stats;
    int out_fmt;           // cg_out_format
};
void run_queries(Graph& G, const QueryCall& c, cudaStream_t s, std::vector<cg_stats>* stats);

// engine_batch.cu
int pass_width(const Graph& G, int kind);  // queries per batched-engine pass for `kind` (1: single-query engine)
int batch_width();  // B of the batched engine (CG_BATCH env: 8 / 16 / 32; anything else disables it)
void run_queries_batched(Graph& G, const QueryCall& c, int B, cudaStream_t s, std::vector<cg_stats>* stats);

// core_graph.cu
void build_core_partial(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs, uint64_t seed,
                        int32_t hub_begin, int32_t hub_end, uint8_t* flags, cudaStream_t s);
void build_core_from_flags(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs, uint64_t seed,
                           const uint8_t* flags, int connectivity, cudaStream_t s);
void save_core(Graph& G, int kind, const char* path, cudaStream_t s);
void export_core_flags(Graph& G, const Core& C, uint8_t* flags, cudaStream_t s);  // u8[m] from the bitmap
void ensure_wcc_graphs(Graph& G, bool two_phase, cudaStream_t s);  // G ∪ G^R, CG ∪ CG^R for WCC
void load_core(Graph& G, int kind, const char* path, cudaStream_t s);
void build_core(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs, uint64_t seed, int alg,
                int connectivity, cudaStream_t s);

// gen.cu
void rmat_generate(uint64_t n, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max, uint64_t seed, int permute,
                   uint64_t e0, uint64_t count, uint32_t* src, uint32_t* dst, uint32_t* w, cudaStream_t s);

}  // namespace cgb
