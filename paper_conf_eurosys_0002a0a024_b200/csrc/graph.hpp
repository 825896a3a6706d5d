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

struct GraphView {
    const uint32_t* ptr;
    const uint32_t* adj;
    const uint2* adjw;
};

inline GraphView view(const Adj& a) { return GraphView{a.ptr.get(), a.adj.get(), a.adjw.get()}; }

struct Core {
    bool built = false;
    int alg = 0;           // 1 = Algorithm 1 (specialized), 2 = Algorithm 2 (general)
    int connectivity = 0;
    Adj adj;               // CG(V, E_c) in the engine layout
    DevBuf<uint8_t> flags; // E_c membership in G's CSR edge order
    std::vector<uint32_t> hubs;
    float build_ms = 0.f;
    // NEXT-1 certificates (Theorem 1 P:1321-1371 and its bottleneck analogs): the Identify
    // queries' values kept as rows hub_vals[v][0..2K) = (Q(h_k) on G at v | Q(h_k) on G^R at v)
    DevBuf<uint32_t> hub_vals;
    uint32_t hub_k = 0;
    Adj rest;              // G minus the CG (phase 2's first sweep, reading N7)
    bool rest_built = false;
    Adj sym;               // WCC: CG ∪ CG^R (built on the first WCC 2Phase query)
    bool sym_built = false;
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
};

inline int core_slot(int kind) { return (kind == CG_BFS || kind == CG_WCC) ? CG_REACH : kind; }

// graph_build.cu
void build_graph(Graph& G, int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                 cudaStream_t s);
void export_adj(const Graph& G, const Adj& a, int64_t* ptr, uint32_t* idx, uint32_t* w, cudaStream_t s);

// engine.cu
struct QueryCall {
    int kind;
    Adj* full_adj;         // G (or G^R for backward Identify queries)
    Adj* core_adj;         // CG (phase 1); ignored when two_phase == 0
    int two_phase;
    const uint32_t* srcs;  // device
    int32_t n_src;
    uint32_t* out;         // n_src * n
    uint32_t* p1;          // nullable
    bool want_stats;
};
void run_queries(Graph& G, const QueryCall& c, cudaStream_t s, std::vector<cg_stats>* stats);

// engine_batch.cu
int batch_width();  // B of the batched engine (CG_BATCH env: 8 / 16 / 32; anything else disables it)
void run_queries_batched(Graph& G, const QueryCall& c, int B, cudaStream_t s, std::vector<cg_stats>* stats);

// core_graph.cu
void build_core_partial(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs, uint64_t seed,
                        int32_t hub_begin, int32_t hub_end, uint8_t* flags, cudaStream_t s);
void build_core_from_flags(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs, uint64_t seed,
                           const uint8_t* flags, int connectivity, cudaStream_t s);
void save_core(Graph& G, int kind, const char* path, cudaStream_t s);
void ensure_wcc_graphs(Graph& G, bool two_phase, cudaStream_t s);  // G ∪ G^R, CG ∪ CG^R for WCC
void load_core(Graph& G, int kind, const char* path, cudaStream_t s);
void build_core(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs, uint64_t seed, int alg,
                int connectivity, cudaStream_t s);

// gen.cu
void rmat_generate(uint64_t n, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max, uint64_t seed, int permute,
                   uint64_t e0, uint64_t count, uint32_t* src, uint32_t* dst, uint32_t* w, cudaStream_t s);

}  // namespace cgb
