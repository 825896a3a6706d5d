// core_graph.cu — Core Graph construction on the GPU (SURVEY §8(a) rows a3-a7, a5').
//
//   a3 hub selection: K highest total-degree vertices, ties to the smaller id (P:464-466,
//      P:1669-1677, reading Q7), or K sampled / given ids (north_star, reading D2).
//   a4 Identify queries (Alg 1 l.3-7): forward Q(h) on G and backward Q(h) on
//      G^R for every hub, run by the same persistent relaxation kernel (FULL mode).
//   a5 tight-edge marking (Alg 1 l.15-25) evaluated directly on G's CSR rows:
//      forward  e(u,v): reached_f(u) && Val_f(u) (+) w == Val_f(v)
//      backward e(u,v): reached_b(v) && Val_b(v) (+) w == Val_b(u)   (the G^R edge v->u,
//      reversed back into G's orientation, l.21), so no edge-id map is needed.
//   a5' Algorithm 2 for BFS / REACH: exact emulation of the sequential FIFO
//      traversals with a shared Qid[] — level-synchronous, each newly labeled vertex's
//      discovering edge is the minimum (FIFO rank of parent, position in parent's row),
//      which is the edge the FIFO examines first; the next level is ordered by that key.
//   a6 connectivity edges (Alg 1 l.8-12; reading Q8).
//   a7 stream compaction of the flagged edges into the CG's CSR.
#include <cub/device/device_scan.cuh>

#include <chrono>
#include <cstdio>
#include <string>
#include <cstring>

#include "graph.hpp"

namespace cgb {

namespace {

constexpr int TB = 256;
constexpr uint32_t FULLM = 0xffffffffu;

inline int grid_rows(uint64_t rows) {
    uint64_t warps = rows;
    uint64_t g = (warps * 32 + TB - 1) / TB;
    if (g > 65536) g = 65536;
    return (int)(g ? g : 1);
}

template <int KIND> struct K;
template <> struct K<CG_SSSP> {
    static constexpr uint32_t INIT = 0xffffffffu;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) { return a + w; }
};
template <> struct K<CG_SSWP> {
    static constexpr uint32_t INIT = 0u;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) { return min(a, w); }
};
template <> struct K<CG_SSNP> {
    static constexpr uint32_t INIT = 0xffffffffu;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) { return max(a, w); }
};
template <> struct K<CG_VITERBI> {
    static constexpr uint32_t INIT = 0u;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) {
        return __float_as_uint(__fdiv_rn(__uint_as_float(a), __uint2float_rn(w)));
    }
};
template <> struct K<CG_BFS> {
    static constexpr uint32_t INIT = 0xffffffffu;
    __device__ static uint32_t ext(uint32_t a, uint32_t) { return a + 1u; }
};
template <> struct K<CG_REACH> {
    static constexpr uint32_t INIT = 0u;
    __device__ static uint32_t ext(uint32_t a, uint32_t) { return a; }
};

__device__ __forceinline__ void edge_at(const GraphView& g, uint32_t e, uint32_t dbits, uint32_t& d, uint32_t& w) {
    if (g.adj) {
        uint32_t x = g.adj[e];
        d = dbits >= 32 ? x : (x & ((1u << dbits) - 1u));
        w = (x >> dbits) + 1u;
    } else {
        uint2 x = g.adjw[e];
        d = x.x;
        w = x.y;
    }
}

// ---------------------------------------------------------------- a3: hubs
__global__ void k_degree_key_max(uint32_t n, const uint32_t* __restrict__ ptr, const uint32_t* __restrict__ rptr,
                                 const unsigned long long* __restrict__ bound, unsigned long long* __restrict__ out) {
    const unsigned long long lim = *bound;
    unsigned long long best = 0;
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
        const unsigned long long deg = (unsigned long long)(ptr[v + 1] - ptr[v]) + (rptr[v + 1] - rptr[v]);
        const unsigned long long key = (deg << 32) | (0xffffffffull - v);  // larger degree, then smaller id
        if (key < lim && key > best) best = key;
    }
    for (int o = 16; o > 0; o >>= 1) {
        unsigned long long y = __shfl_xor_sync(FULLM, best, o);
        best = y > best ? y : best;
    }
    if ((threadIdx.x & 31) == 0 && best) atomicMax(out, best);
}

// ---------------------------------------------------------------- a5: Alg 1 marking
// Warp per row u of G; hubs [0, nh) of the current group; valf/valb: nh x n values.
template <int KIND>
__global__ void k_mark_tight(uint32_t n, GraphView g, uint32_t dbits, int nh, const uint32_t* __restrict__ valf,
                             const uint32_t* __restrict__ valb, uint8_t* __restrict__ flags) {
    using O = K<KIND>;
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u < n; u += nw) {
        const uint32_t r0 = g.ptr[u], r1 = g.ptr[u + 1];
        for (uint32_t e = r0 + lane; e < r1; e += 32) {
            uint32_t v, w;
            edge_at(g, e, dbits, v, w);
            bool tight = false;
            for (int k = 0; k < nh && !tight; ++k) {
                const uint32_t* vf = valf + (size_t)k * n;
                const uint32_t* vb = valb + (size_t)k * n;
                const uint32_t fu = vf[u];
                if (fu != O::INIT && O::ext(fu, w) == vf[v]) tight = true;   // l.16-19, d == f
                const uint32_t bv = vb[v];
                if (bv != O::INIT && O::ext(bv, w) == vb[u]) tight = true;   // l.16-21, d == b
            }
            if (tight) flags[e] = 1;
        }
    }
}

// ---------------------------------------------------------------- a6: connectivity
// kind_sel: 0 = min weight (SSSP/SSNP/Viterbi), 1 = max weight (SSWP), 2 = first edge.
__global__ void k_connectivity(uint32_t n, GraphView g, uint32_t dbits, int kind_sel, uint8_t* __restrict__ flags) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u < n; u += nw) {
        const uint32_t r0 = g.ptr[u], r1 = g.ptr[u + 1];
        if (r0 == r1) continue;
        bool any = false;
        unsigned long long best = ~0ull;
        for (uint32_t e = r0 + lane; e < r1; e += 32) {
            any |= flags[e] != 0;
            uint32_t v, w;
            edge_at(g, e, dbits, v, w);
            const uint32_t wk = kind_sel == 0 ? w : (kind_sel == 1 ? ~w : 0u);
            const unsigned long long key = ((unsigned long long)wk << 32) | (e - r0);
            best = key < best ? key : best;
        }
        if (__any_sync(FULLM, any)) continue;
        for (int o = 16; o > 0; o >>= 1) {
            unsigned long long y = __shfl_xor_sync(FULLM, best, o);
            best = y < best ? y : best;
        }
        if (lane == 0) flags[r0 + (uint32_t)best] = 1;
    }
}

// ---------------------------------------------------------------- a7: split rows
// E_c membership bits (bit e of word e/32) from the u8 marks: thread per word, coalesced
__global__ void k_pack_bits(uint64_t m, const uint8_t* __restrict__ flags, uint32_t* __restrict__ bits) {
    for (uint64_t wi = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; wi < (m + 31) / 32;
         wi += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t x = 0;
        for (uint32_t b = 0; b < 32 && wi * 32 + b < m; ++b) x |= (uint32_t)(flags[wi * 32 + b] != 0) << b;
        bits[wi] = x;
    }
}

__global__ void k_unpack_bits(uint64_t m, const uint32_t* __restrict__ bits, uint8_t* __restrict__ flags) {
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x)
        flags[e] = (bits[e >> 5] >> (e & 31)) & 1u;
}

__device__ __forceinline__ bool bit_at(const uint32_t* __restrict__ bits, uint32_t e) { return (bits[e >> 5] >> (e & 31)) & 1u; }

// Split-CSR layout (graph.hpp Core): warp per row u of G; the row's CG edges are
// copied to [ptr[u], cg_end[u]) and the others to [cg_end[u], ptr[u+1]), both in canonical
// order (stable partition); *mcg accumulates |E_c|.
__global__ void k_split_rows(uint32_t n, const uint32_t* __restrict__ ptr, const uint32_t* __restrict__ bits,
                             const uint32_t* __restrict__ adj, const uint2* __restrict__ adjw,
                             uint32_t* __restrict__ sadj, uint2* __restrict__ sadjw, uint32_t* __restrict__ cg_end,
                             unsigned long long* __restrict__ mcg) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t lt = (1u << lane) - 1u;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    unsigned long long tot = 0;
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u < n; u += nw) {
        const uint32_t r0 = ptr[u], r1 = ptr[u + 1];
        uint32_t c = 0;
        for (uint32_t b = r0; b < r1; b += 32) c += __popc(__ballot_sync(FULLM, b + lane < r1 && bit_at(bits, b + lane)));
        const uint32_t ce = r0 + c;
        uint32_t oc = r0, orr = ce;
        for (uint32_t b = r0; b < r1; b += 32) {
            const uint32_t e = b + lane;
            const bool in = e < r1;
            const bool f = in && bit_at(bits, e);
            const uint32_t bc = __ballot_sync(FULLM, f), br = __ballot_sync(FULLM, in && !f);
            if (in) {
                const uint32_t p = f ? oc + __popc(bc & lt) : orr + __popc(br & lt);
                if (adj) sadj[p] = adj[e]; else sadjw[p] = adjw[e];
            }
            oc += __popc(bc);
            orr += __popc(br);
        }
        if (lane == 0) cg_end[u] = ce;
        tot += c;
    }
    if (lane == 0 && tot) atomicAdd(mcg, tot);
}

// ---------------------------------------------------------------- a5': Alg 2
// Expand level L (FIFO order = list order) of a traversal labeled `lab`.
template <bool REV>
__global__ void k_alg2_expand(GraphView g, uint32_t dbits, const uint32_t* __restrict__ L, uint32_t nl,
                              const uint32_t* __restrict__ qid, uint32_t lab, unsigned long long* __restrict__ key,
                              uint8_t* __restrict__ flags, const uint32_t* __restrict__ reid) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t r = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); r < nl; r += nw) {
        const uint32_t u = L[r];
        const uint32_t r0 = g.ptr[u], r1 = g.ptr[u + 1];
        for (uint32_t e = r0 + lane; e < r1; e += 32) {
            uint32_t v, w;
            edge_at(g, e, dbits, v, w);
            const uint32_t q = qid[v];
            if (q == lab) continue;                        // l.16: Qid(v) == s -> skip
            if (q == 0)                                    // l.19: first examiner in FIFO order wins
                atomicMin(key + v, ((unsigned long long)r << 32) | (e - r0));
            else                                           // l.18: add e(u,v), v labeled elsewhere
                flags[REV ? reid[e] : e] = 1;
        }
    }
}

__device__ __forceinline__ bool alg2_winner(const uint32_t* qid, const unsigned long long* key, uint32_t v, uint64_t r,
                                            uint32_t j) {
    return qid[v] == 0 && key[v] == ((((unsigned long long)r) << 32) | j);
}

template <bool EMIT, bool REV>
__global__ void k_alg2_winners(GraphView g, uint32_t dbits, const uint32_t* __restrict__ L, uint32_t nl, uint32_t* qid,
                               uint32_t lab, unsigned long long* key, uint32_t* __restrict__ cnt,
                               const uint32_t* __restrict__ base, uint32_t* __restrict__ next,
                               uint8_t* __restrict__ flags, const uint32_t* __restrict__ reid) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t r = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); r < nl; r += nw) {
        const uint32_t u = L[r];
        const uint32_t r0 = g.ptr[u], r1 = g.ptr[u + 1];
        uint32_t o = EMIT ? base[r] : 0u;
        for (uint32_t b = r0; b < r1; b += 32) {
            const uint32_t e = b + lane;
            uint32_t v = 0, w;
            bool win = false;
            if (e < r1) {
                edge_at(g, e, dbits, v, w);
                win = alg2_winner(qid, key, v, r, e - r0);
            }
            const uint32_t bal = __ballot_sync(FULLM, win);
            if (EMIT && win) {
                next[o + __popc(bal & ((1u << lane) - 1u))] = v;   // l.20 Fifo.push(v)
                flags[REV ? reid[e] : e] = 1;                      // l.18 add e(u,v)
            }
            o += __popc(bal);
            __syncwarp();
            if (EMIT && win) {                                     // l.21 Qid(v) <- s
                qid[v] = lab;
                key[v] = ~0ull;
            }
        }
        if (!EMIT && lane == 0) cnt[r] = o;
    }
}

void exclusive_sum(const uint32_t* in, uint32_t* out, uint64_t m, cudaStream_t s) {
    size_t tmp = 0;
    CGB_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, in, out, (int64_t)m, s));
    DevBuf<uint8_t> t(tmp, s);
    CGB_CUDA(cub::DeviceScan::ExclusiveSum(t.get(), tmp, in, out, (int64_t)m, s));
    count_launch(2);
}

std::vector<uint32_t> select_hubs(Graph& G, int32_t K, int policy, const uint32_t* given, uint64_t seed,
                                  cudaStream_t s) {
    std::vector<uint32_t> hubs;
    if (policy == CG_HUBS_GIVEN) {
        CGB_CHECK(given != nullptr, CG_EINVAL, "CG_HUBS_GIVEN needs a host hub array");
        for (int k = 0; k < K; ++k) {
            CGB_CHECK(given[k] < G.n, CG_EINVAL, "hub id >= n");
            hubs.push_back(given[k]);
        }
        return hubs;
    }
    if (policy == CG_HUBS_SAMPLED) {
        // uniform over vertices with outdeg > 0, distinct, splitmix64(seed + i) draws
        std::vector<uint32_t> ptr(G.n + 1);
        CGB_CUDA(cudaMemcpyAsync(ptr.data(), G.g.ptr.get(), 4ull * (G.n + 1), cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaStreamSynchronize(s));
        std::vector<uint32_t> cand;
        for (uint32_t v = 0; v < G.n; ++v)
            if (ptr[v + 1] > ptr[v]) cand.push_back(v);
        CGB_CHECK((int64_t)cand.size() >= K, CG_EINVAL, "fewer than K vertices with outdeg > 0");
        std::vector<uint8_t> taken(cand.size(), 0);
        for (uint64_t i = 0; (int)hubs.size() < K; ++i) {
            uint64_t x = seed + i * 0x9E3779B97F4A7C15ull;
            x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
            x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
            x ^= x >> 31;
            const uint64_t j = x % cand.size();
            if (!taken[j]) { taken[j] = 1; hubs.push_back(cand[j]); }
        }
        return hubs;
    }
    CGB_CHECK(policy == CG_HUBS_TOPDEG, CG_EINVAL, "bad hub policy");
    DevBuf<unsigned long long> keys(K + 1, s);
    const unsigned long long top = ~0ull;
    CGB_CUDA(cudaMemsetAsync(keys.get(), 0, (K + 1) * 8ull, s));
    CGB_CUDA(cudaMemcpyAsync(keys.get(), &top, 8, cudaMemcpyHostToDevice, s));
    for (int k = 0; k < K; ++k)
        CGB_LAUNCH(k_degree_key_max, 296, TB, 0, s, G.n, G.g.ptr.get(), G.gr.ptr.get(), keys.get() + k,
                   keys.get() + k + 1);
    std::vector<unsigned long long> h(K + 1);
    CGB_CUDA(cudaMemcpyAsync(h.data(), keys.get(), (K + 1) * 8ull, cudaMemcpyDeviceToHost, s));
    CGB_CUDA(cudaStreamSynchronize(s));
    for (int k = 1; k <= K; ++k) hubs.push_back((uint32_t)(0xffffffffull - (h[k] & 0xffffffffull)));
    return hubs;
}

template <int KIND>
void mark_group(Graph& G, int nh, const uint32_t* vf, const uint32_t* vb, uint8_t* flags, cudaStream_t s) {
    CGB_LAUNCH(k_mark_tight<KIND>, grid_rows(G.n), TB, 0, s, G.n, view(G.g), G.dbits, nh, vf, vb, flags);
}

// hub rows for the NEXT-1 certificates (row stride 2*KP, KP = K rounded up to 4 so that the
// engine reads 16 B chunks): HB[v][k0+j] = vf[j][v], HB[v][KP+k0+j] = vb[j][v]
__global__ void k_hub_rows(uint32_t n, int nh, int k0, int KP, const uint32_t* __restrict__ vf,
                           const uint32_t* __restrict__ vb, uint32_t* __restrict__ hb) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < (uint64_t)n * nh;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t j = (uint32_t)(i / n), v = (uint32_t)(i % n);
        hb[(size_t)v * 2 * KP + k0 + j] = vf[(size_t)j * n + v];
        hb[(size_t)v * 2 * KP + KP + k0 + j] = vb[(size_t)j * n + v];
    }
}

void alg1(Graph& G, int kind, const std::vector<uint32_t>& hubs, uint8_t* flags, Core& C, cudaStream_t s) {
    const int K = (int)hubs.size();
    // certificates are kept for the kinds that have one (SSSP, SSWP, SSNP) and K <= 64
    const bool keep = (kind == CG_SSSP || kind == CG_SSWP || kind == CG_SSNP) && K <= 64;
    C.hub_vals.reset();
    C.hub_k = 0;
    const int KP = (K + 3) & ~3;
    if (keep) {
        C.hub_vals.alloc((size_t)G.n * 2 * KP, s);
        C.hub_k = (uint32_t)K;
    }
    const int group = K < 16 ? K : 16;
    DevBuf<uint32_t> hsrc(K, s);
    CGB_CUDA(cudaMemcpyAsync(hsrc.get(), hubs.data(), 4ull * K, cudaMemcpyHostToDevice, s));
    DevBuf<uint32_t> vf((size_t)group * G.n, s), vb((size_t)group * G.n, s);
    for (int k0 = 0; k0 < K; k0 += group) {
        const int nh = (K - k0) < group ? (K - k0) : group;
        QueryCall f{kind, view(G.g), view(G.g), GraphView{}, nullptr, 0, hsrc.get() + k0, nh, vf.get(), nullptr,
                    false, CG_OUT_U32};
        run_queries(G, f, s, nullptr);                   // Alg 1 l.4: Identify(G, forward)
        QueryCall b{kind, view(G.gr), view(G.gr), GraphView{}, nullptr, 0, hsrc.get() + k0, nh, vb.get(), nullptr,
                    false, CG_OUT_U32};
        run_queries(G, b, s, nullptr);                   // Alg 1 l.5: Identify(G^R, backward)
        switch (kind) {
        case CG_SSSP: mark_group<CG_SSSP>(G, nh, vf.get(), vb.get(), flags, s); break;
        case CG_SSWP: mark_group<CG_SSWP>(G, nh, vf.get(), vb.get(), flags, s); break;
        case CG_SSNP: mark_group<CG_SSNP>(G, nh, vf.get(), vb.get(), flags, s); break;
        case CG_VITERBI: mark_group<CG_VITERBI>(G, nh, vf.get(), vb.get(), flags, s); break;
        case CG_BFS: mark_group<CG_BFS>(G, nh, vf.get(), vb.get(), flags, s); break;
        case CG_REACH: mark_group<CG_REACH>(G, nh, vf.get(), vb.get(), flags, s); break;
        }
        if (keep)
            CGB_LAUNCH(k_hub_rows, 4096, TB, 0, s, G.n, nh, k0, KP, vf.get(), vb.get(), C.hub_vals.get());
    }
}

void alg2(Graph& G, const std::vector<uint32_t>& hubs, uint8_t* flags, bool per_direction, cudaStream_t s) {
    const uint32_t n = G.n;
    // reading Q9: one Qid[] shared by the forward and backward traversals (literal Alg 2), or
    // one per direction (CG_ALG_GENERAL_PERDIR)
    DevBuf<uint32_t> qid(per_direction ? 2ull * n : n, s), la(n + 1, s), lb(n + 1, s), cnt(n + 1, s), base(n + 1, s);
    DevBuf<unsigned long long> key(n, s);
    CGB_CUDA(cudaMemsetAsync(qid.get(), 0, qid.bytes(), s));
    CGB_CUDA(cudaMemsetAsync(key.get(), 0xff, 8ull * n, s));
    for (size_t k = 0; k < hubs.size(); ++k) {               // Alg 2 l.5
        const uint32_t lab = (uint32_t)k + 1;                 // reading Q10
        for (int dir = 0; dir < 2; ++dir) {                   // l.6 on G, l.7 on G^R
            const GraphView g = dir == 0 ? view(G.g) : view(G.gr);
            uint32_t* Q = qid.get() + (per_direction && dir == 1 ? n : 0);
            uint32_t* L = la.get();
            uint32_t* N = lb.get();
            uint32_t nl = 1;
            CGB_CUDA(cudaMemcpyAsync(L, &hubs[k], 4, cudaMemcpyHostToDevice, s));   // l.12
            while (nl) {                                                          // l.13
                const int grid = grid_rows(nl);
                if (dir == 0) {
                    CGB_LAUNCH(k_alg2_expand<false>, grid, TB, 0, s, g, G.dbits, L, nl, Q, lab, key.get(),
                               flags, (const uint32_t*)nullptr);
                    CGB_LAUNCH((k_alg2_winners<false, false>), grid, TB, 0, s, g, G.dbits, L, nl, Q, lab,
                               key.get(), cnt.get(), (const uint32_t*)nullptr, (uint32_t*)nullptr, flags,
                               (const uint32_t*)nullptr);
                } else {
                    CGB_LAUNCH(k_alg2_expand<true>, grid, TB, 0, s, g, G.dbits, L, nl, Q, lab, key.get(),
                               flags, G.reid.get());
                    CGB_LAUNCH((k_alg2_winners<false, true>), grid, TB, 0, s, g, G.dbits, L, nl, Q, lab,
                               key.get(), cnt.get(), (const uint32_t*)nullptr, (uint32_t*)nullptr, flags,
                               G.reid.get());
                }
                CGB_CUDA(cudaMemsetAsync(cnt.get() + nl, 0, 4, s));
                exclusive_sum(cnt.get(), base.get(), (uint64_t)nl + 1, s);
                uint32_t total = 0;
                CGB_CUDA(cudaMemcpyAsync(&total, base.get() + nl, 4, cudaMemcpyDeviceToHost, s));
                CGB_CUDA(cudaStreamSynchronize(s));
                if (total) {
                    if (dir == 0)
                        CGB_LAUNCH((k_alg2_winners<true, false>), grid, TB, 0, s, g, G.dbits, L, nl, Q, lab,
                                   key.get(), cnt.get(), base.get(), N, flags, (const uint32_t*)nullptr);
                    else
                        CGB_LAUNCH((k_alg2_winners<true, true>), grid, TB, 0, s, g, G.dbits, L, nl, Q, lab,
                                   key.get(), cnt.get(), base.get(), N, flags, G.reid.get());
                }
                uint32_t* t = L; L = N; N = t;
                nl = total;
            }
        }
    }
}

}  // namespace

namespace {

// ---------------------------------------------------------------- CG^R (phase-1 pull)
__global__ void k_cg_indeg(uint32_t n, GraphView cg, uint32_t dbits, uint32_t* __restrict__ indeg) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u < n; u += nw)
        for (uint32_t e = cg.ptr[u] + lane; e < cg.end[u]; e += 32) {
            uint32_t v, w;
            edge_at(cg, e, dbits, v, w);
            atomicAdd(indeg + v, 1u);
        }
}

// CG^R rows: in-edge (u -> v, w) stored in row v as u in G's edge encoding (order within a row is
// immaterial: the pull's select is order-independent)
__global__ void k_cg_rfill(uint32_t n, GraphView cg, uint32_t dbits, int packed, const uint32_t* __restrict__ rptr,
                           uint32_t* __restrict__ fill, uint32_t* __restrict__ radj, uint2* __restrict__ radjw) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u < n; u += nw)
        for (uint32_t e = cg.ptr[u] + lane; e < cg.end[u]; e += 32) {
            uint32_t v, w;
            edge_at(cg, e, dbits, v, w);
            const uint32_t pos = rptr[v] + atomicAdd(fill + v, 1u);
            if (packed) radj[pos] = (uint32_t)u | ((w - 1u) << dbits);
            else radjw[pos] = make_uint2((uint32_t)u, w);
        }
}

// the vertices with in-edges, in vertex order, and their first in-edge (flags -> positions)
__global__ void k_pull_list(uint32_t n, const uint32_t* __restrict__ rptr, const uint32_t* __restrict__ pos,
                            uint32_t* __restrict__ lv, uint32_t* __restrict__ lo) {
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        if (rptr[v + 1] > rptr[v]) {
            lv[pos[v]] = (uint32_t)v;
            lo[pos[v]] = rptr[v];
        }
}

__global__ void k_has_in(uint32_t n, const uint32_t* __restrict__ indeg, uint32_t* __restrict__ flag) {
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v <= n; v += (uint64_t)gridDim.x * blockDim.x)
        flag[v] = v < n && indeg[v] ? 1u : 0u;
}

void build_pull(Graph& G, Core& C, cudaStream_t s) {
    const GraphView cg = core_view(G, C);
    DevBuf<uint32_t> indeg(G.n + 1, s), pos(G.n + 1, s);
    CGB_CUDA(cudaMemsetAsync(indeg.get(), 0, indeg.bytes(), s));
    CGB_LAUNCH(k_cg_indeg, grid_rows(G.n), TB, 0, s, G.n, cg, G.dbits, indeg.get());
    C.rcg.n = G.n;
    C.rcg.m = C.m_cg;
    C.rcg.ptr.alloc(G.n + 1, s);
    exclusive_sum(indeg.get(), C.rcg.ptr.get(), (uint64_t)G.n + 1, s);  // indeg[n] = 0
    C.rcg.adj.reset();
    C.rcg.adjw.reset();
    if (G.packed) C.rcg.adj.alloc(adj_alloc_elems(C.m_cg, 4), s); else C.rcg.adjw.alloc(adj_alloc_elems(C.m_cg, 8), s);
    CGB_LAUNCH(k_has_in, 4 * G.num_sms, TB, 0, s, G.n, indeg.get(), pos.get());
    DevBuf<uint32_t> flag(G.n + 1, s);
    CGB_CUDA(cudaMemcpyAsync(flag.get(), pos.get(), 4ull * (G.n + 1), cudaMemcpyDeviceToDevice, s));
    exclusive_sum(flag.get(), pos.get(), (uint64_t)G.n + 1, s);
    CGB_CUDA(cudaMemsetAsync(indeg.get(), 0, indeg.bytes(), s));  // reused as the fill counters
    CGB_LAUNCH(k_cg_rfill, grid_rows(G.n), TB, 0, s, G.n, cg, G.dbits, G.packed ? 1 : 0, C.rcg.ptr.get(), indeg.get(),
               C.rcg.adj.get(), C.rcg.adjw.get());
    uint32_t cnt = 0;
    CGB_CUDA(cudaMemcpyAsync(&cnt, pos.get() + G.n, 4, cudaMemcpyDeviceToHost, s));
    CGB_CUDA(cudaStreamSynchronize(s));
    C.pl_count = cnt;
    C.pl_v.alloc(cnt + 1, s);
    C.pl_lo.alloc(cnt + 1, s);
    CGB_LAUNCH(k_pull_list, 4 * G.num_sms, TB, 0, s, G.n, C.rcg.ptr.get(), pos.get(), C.pl_v.get(), C.pl_lo.get());
    CGB_CUDA(cudaStreamSynchronize(s));
    C.rcg_built = true;
}

// a7: the split rows from C.fbits
void split_core(Graph& G, Core& C, cudaStream_t s) {
    C.rcg_built = false;
    C.cg_end.alloc(G.n ? G.n : 1, s);
    C.sadj.reset();
    C.sadjw.reset();
    if (G.packed) C.sadj.alloc(adj_alloc_elems(G.m, 4), s); else C.sadjw.alloc(adj_alloc_elems(G.m, 8), s);
    DevBuf<unsigned long long> mcg(1, s);
    CGB_CUDA(cudaMemsetAsync(mcg.get(), 0, 8, s));
    CGB_LAUNCH(k_split_rows, grid_rows(G.n), TB, 0, s, G.n, G.g.ptr.get(), C.fbits.get(), G.g.adj.get(), G.g.adjw.get(),
               C.sadj.get(), C.sadjw.get(), C.cg_end.get(), mcg.get());
    unsigned long long h = 0;
    CGB_CUDA(cudaMemcpyAsync(&h, mcg.get(), 8, cudaMemcpyDeviceToHost, s));
    CGB_CUDA(cudaStreamSynchronize(s));
    C.m_cg = (uint32_t)h;
    build_pull(G, C, s);
}

// a6 + a7: connectivity edges (Alg 1 l.8-12) on the u8 marks (device, m bytes, consumed),
// then the membership bitmap and the split rows (graph.hpp Core)
void finalize_core(Graph& G, int kind, Core& C, int connectivity, uint8_t* marks, cudaStream_t s) {
    if (G.m && connectivity) {
        const int sel = (kind == CG_SSWP) ? 1 : ((kind == CG_BFS || kind == CG_REACH) ? 2 : 0);
        CGB_LAUNCH(k_connectivity, grid_rows(G.n), TB, 0, s, G.n, view(G.g), G.dbits, sel, marks);
    }
    C.fbits.alloc(((size_t)G.m + 31) / 32 + 1, s);
    if (G.m) CGB_LAUNCH(k_pack_bits, 4 * G.num_sms, TB, 0, s, (uint64_t)G.m, marks, C.fbits.get());
    split_core(G, C, s);
}

struct Timer {
    cudaEvent_t e0, e1;
    cudaStream_t s;
    explicit Timer(cudaStream_t st) : s(st) {
        CGB_CUDA(cudaEventCreate(&e0));
        CGB_CUDA(cudaEventCreate(&e1));
        CGB_CUDA(cudaEventRecord(e0, s));
    }
    float stop() {
        CGB_CUDA(cudaEventRecord(e1, s));
        CGB_CUDA(cudaEventSynchronize(e1));
        float ms = 0.f;
        CGB_CUDA(cudaEventElapsedTime(&ms, e0, e1));
        return ms;
    }
    ~Timer() {
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
    }
};

bool alg1_kind(int kind) { return kind == CG_SSSP || kind == CG_SSWP || kind == CG_SSNP || kind == CG_VITERBI; }

// order-independent 64-bit fingerprint of the canonical graph (row offsets and edge words)
__device__ __forceinline__ unsigned long long mix64(unsigned long long x) {
    x ^= x >> 30;
    x *= 0xbf58476d1ce4e5b9ull;
    x ^= x >> 27;
    x *= 0x94d049bb133111ebull;
    return x ^ (x >> 31);
}
__global__ void k_graph_hash(uint32_t n, uint32_t m, const uint32_t* __restrict__ ptr, const uint32_t* __restrict__ adj,
                             const uint2* __restrict__ adjw, unsigned long long* out) {
    unsigned long long h = 0;
    const uint64_t tot = (uint64_t)n + 1 + m;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < tot; i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long x;
        if (i <= n) x = ptr[i];
        else if (adj) x = adj[i - n - 1];
        else x = ((unsigned long long)adjw[i - n - 1].x << 32) | adjw[i - n - 1].y;
        h += mix64(i * 0x9e3779b97f4a7c15ull ^ x);
    }
    for (int o = 16; o > 0; o >>= 1) h += __shfl_xor_sync(0xffffffffu, h, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(out, h);
}

unsigned long long graph_hash(Graph& G, cudaStream_t s) {
    DevBuf<unsigned long long> d(1, s);
    CGB_CUDA(cudaMemsetAsync(d.get(), 0, 8, s));
    CGB_LAUNCH(k_graph_hash, 4 * G.num_sms, TB, 0, s, G.n, G.m, G.g.ptr.get(), G.g.adj.get(), G.g.adjw.get(), d.get());
    unsigned long long h = 0;
    CGB_CUDA(cudaMemcpyAsync(&h, d.get(), 8, cudaMemcpyDeviceToHost, s));
    CGB_CUDA(cudaStreamSynchronize(s));
    return h;
}

struct CoreFileHeader {  // cg_core_save / cg_core_load (little-endian)
    char magic[8];       // "CGB200\0\1"
    uint32_t version, kind, alg, connectivity, K, n, m, reserved;
    unsigned long long graph_hash, m_cg;
};
const char kMagic[8] = {'C', 'G', 'B', '2', '0', '0', 0, 1};

}  // namespace

void build_core(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs_in, uint64_t seed, int alg,
                int connectivity, cudaStream_t s) {
    CGB_CHECK(kind >= 0 && kind <= CG_WCC, CG_EINVAL, "bad kind");
    CGB_CHECK(K > 0 && (uint32_t)K <= G.n, CG_EINVAL, "K must be in [1, n]");
    if (kind == CG_WCC) kind = CG_REACH;  // WCC uses REACH's general CG; its G ∪ G^R is made per query
    // reading Q9': the general CG keeps one Qid[] per traversal direction by default
    if (alg == CG_ALG_AUTO) alg = (kind == CG_BFS || kind == CG_REACH) ? CG_ALG_GENERAL_PERDIR : CG_ALG_SPECIALIZED;
    CGB_CHECK(alg == CG_ALG_SPECIALIZED || alg == CG_ALG_GENERAL || alg == CG_ALG_GENERAL_PERDIR, CG_EINVAL,
              "bad CG algorithm");
    if (connectivity < 0) connectivity = (alg == CG_ALG_SPECIALIZED) ? 1 : 0;  // reading Q11

    Timer t(s);
    std::vector<uint32_t> hubs = select_hubs(G, K, policy, hubs_in, seed, s);
    Core& C = G.core[core_slot(kind)];
    C.built = false;
    C.sym_built = false;
    C.hub_vals.reset();
    C.hub_k = 0;
    DevBuf<uint8_t> marks(G.m ? G.m : 1, s);  // E_c marks in G's CSR order (u8: racing writers)
    CGB_CUDA(cudaMemsetAsync(marks.get(), 0, marks.bytes(), s));
    if (G.m) {
        if (alg == CG_ALG_SPECIALIZED) alg1(G, kind, hubs, marks.get(), C, s);
        else alg2(G, hubs, marks.get(), alg == CG_ALG_GENERAL_PERDIR, s);
    }
    finalize_core(G, kind, C, connectivity, marks.get(), s);
    C.hubs = hubs;
    C.alg = alg;
    C.connectivity = connectivity;
    C.build_ms = t.stop();
    C.built = true;
}

// ------------------------------------------------------------------ WCC graphs (NEXT-3)
// Row v of the symmetrised graph = v's (flagged) out-edges in G followed by its (flagged)
// in-edges (G^R row v; an in-edge's flag is that of its CSR edge, reid).  Edge words keep G's
// encoding (the WCC EdgeFunction ignores the weight).
__global__ void k_sym_count(uint32_t n, const uint32_t* __restrict__ gp, const uint32_t* __restrict__ rp,
                            const uint32_t* __restrict__ reid, const uint32_t* __restrict__ flags,
                            uint32_t* __restrict__ cnt) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u <= n; u += nw) {
        if (u == n) { if (lane == 0) cnt[n] = 0; continue; }
        uint32_t c = 0;
        if (flags) {
            for (uint32_t e = gp[u] + lane; e < gp[u + 1]; e += 32) c += bit_at(flags, e);
            for (uint32_t e = rp[u] + lane; e < rp[u + 1]; e += 32) c += bit_at(flags, reid[e]);
            for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(FULLM, c, o);
        } else {
            c = (gp[u + 1] - gp[u]) + (rp[u + 1] - rp[u]);
        }
        if (lane == 0) cnt[u] = c;
    }
}

__device__ __forceinline__ void sym_copy_row(uint32_t r0, uint32_t r1, const uint32_t* __restrict__ reid,
                                             const uint32_t* __restrict__ flags, const uint32_t* __restrict__ adj,
                                             const uint2* __restrict__ adjw, uint32_t* __restrict__ sadj,
                                             uint2* __restrict__ sadjw, uint32_t& o) {
    const uint32_t lane = threadIdx.x & 31;
    for (uint32_t b = r0; b < r1; b += 32) {
        const uint32_t e = b + lane;
        const bool f = e < r1 && (!flags || bit_at(flags, reid ? reid[e] : e));
        const uint32_t bal = __ballot_sync(FULLM, f);
        if (f) {
            const uint32_t p = o + __popc(bal & ((1u << lane) - 1u));
            if (adj) sadj[p] = adj[e]; else sadjw[p] = adjw[e];
        }
        o += __popc(bal);
    }
}

__global__ void k_sym_scatter(uint32_t n, const uint32_t* __restrict__ gp, const uint32_t* __restrict__ rp,
                              const uint32_t* __restrict__ reid, const uint32_t* __restrict__ flags,
                              const uint32_t* __restrict__ sp, const uint32_t* __restrict__ gadj,
                              const uint2* __restrict__ gadjw, const uint32_t* __restrict__ radj,
                              const uint2* __restrict__ radjw, uint32_t* __restrict__ sadj, uint2* __restrict__ sadjw) {
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); u < n; u += nw) {
        uint32_t o = sp[u];
        sym_copy_row(gp[u], gp[u + 1], nullptr, flags, gadj, gadjw, sadj, sadjw, o);
        sym_copy_row(rp[u], rp[u + 1], reid, flags, radj, radjw, sadj, sadjw, o);
    }
}

void symmetrize(Graph& G, const uint32_t* flags, Adj& out, cudaStream_t s) {
    DevBuf<uint32_t> cnt(G.n + 1, s);
    CGB_LAUNCH(k_sym_count, grid_rows(G.n + 1), TB, 0, s, G.n, G.g.ptr.get(), G.gr.ptr.get(), G.reid.get(), flags,
               cnt.get());
    out.n = G.n;
    out.ptr.alloc(G.n + 1, s);
    exclusive_sum(cnt.get(), out.ptr.get(), (uint64_t)G.n + 1, s);
    uint32_t ms = 0;
    CGB_CUDA(cudaMemcpyAsync(&ms, out.ptr.get() + G.n, 4, cudaMemcpyDeviceToHost, s));
    CGB_CUDA(cudaStreamSynchronize(s));
    out.m = ms;
    out.adj.reset();
    out.adjw.reset();
    if (G.packed) out.adj.alloc(adj_alloc_elems(ms, 4), s); else out.adjw.alloc(adj_alloc_elems(ms, 8), s);
    CGB_LAUNCH(k_sym_scatter, grid_rows(G.n), TB, 0, s, G.n, G.g.ptr.get(), G.gr.ptr.get(), G.reid.get(), flags,
               out.ptr.get(), G.g.adj.get(), G.g.adjw.get(), G.gr.adj.get(), G.gr.adjw.get(), out.adj.get(),
               out.adjw.get());
    CGB_CUDA(cudaStreamSynchronize(s));
}

void ensure_wcc_graphs(Graph& G, bool two_phase, cudaStream_t s) {
    if (!G.gsym_built) {
        symmetrize(G, nullptr, G.gsym, s);
        G.gsym_built = true;
    }
    Core& C = G.core[CG_REACH];
    if (two_phase && C.built && !C.sym_built) {
        symmetrize(G, C.fbits.get(), C.sym, s);
        C.sym_built = true;
    }
}

// NEXT-4: Algorithm 1 is a union over hubs (each hub's tight edges are marked independently,
// P:757-786), so the 2K Identify queries can be split across GPUs: each rank marks the flags of
// its hub range, the flags are OR-reduced (ncclAllReduce max on u8), and every rank finalises.
// Algorithm 2 is sequential in the hubs (shared labels) and is not split.
void build_core_partial(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs_in, uint64_t seed,
                        int32_t hub_begin, int32_t hub_end, uint8_t* flags, cudaStream_t s) {
    CGB_CHECK(alg1_kind(kind), CG_EUNSUPPORTED, "partial builds need Algorithm 1 (SSSP/SSWP/SSNP/Viterbi)");
    CGB_CHECK(K > 0 && (uint32_t)K <= G.n, CG_EINVAL, "K must be in [1, n]");
    CGB_CHECK(0 <= hub_begin && hub_begin <= hub_end && hub_end <= K, CG_EINVAL, "bad hub range");
    std::vector<uint32_t> hubs = select_hubs(G, K, policy, hubs_in, seed, s);
    if (G.m) CGB_CUDA(cudaMemsetAsync(flags, 0, G.m, s));
    if (G.m && hub_end > hub_begin) {
        std::vector<uint32_t> sub(hubs.begin() + hub_begin, hubs.begin() + hub_end);
        Core scratch;  // no certificates are kept for partial builds
        alg1(G, kind, sub, flags, scratch, s);
    }
    CGB_CUDA(cudaStreamSynchronize(s));
}

void build_core_from_flags(Graph& G, int kind, int32_t K, int policy, const uint32_t* hubs_in, uint64_t seed,
                           const uint8_t* flags, int connectivity, cudaStream_t s) {
    CGB_CHECK(alg1_kind(kind), CG_EUNSUPPORTED, "merged builds need Algorithm 1 (SSSP/SSWP/SSNP/Viterbi)");
    CGB_CHECK(K > 0 && (uint32_t)K <= G.n, CG_EINVAL, "K must be in [1, n]");
    if (connectivity < 0) connectivity = 1;  // reading Q11 for Algorithm 1
    Timer t(s);
    std::vector<uint32_t> hubs = select_hubs(G, K, policy, hubs_in, seed, s);
    Core& C = G.core[core_slot(kind)];
    C.built = false;
    C.sym_built = false;
    C.hub_vals.reset();
    C.hub_k = 0;
    DevBuf<uint8_t> marks(G.m ? G.m : 1, s);  // writable copy (connectivity edges are added)
    if (G.m) CGB_CUDA(cudaMemcpyAsync(marks.get(), flags, G.m, cudaMemcpyDeviceToDevice, s));
    finalize_core(G, kind, C, connectivity, marks.get(), s);
    C.hubs = hubs;
    C.alg = CG_ALG_SPECIALIZED;
    C.connectivity = connectivity;
    C.build_ms = t.stop();
    C.built = true;
}

// NEXT-4 persistence: the CG is identified once for all future queries; the file
// holds its edge flags (bit-packed, G's CSR order), hubs and options, tied to G by n, m and a
// fingerprint of the canonical CSR.
void save_core(Graph& G, int kind, const char* path, cudaStream_t s) {
    const Core& C = G.core[core_slot(kind)];
    CGB_CHECK(C.built, CG_ENOCG, "Core Graph not built for this kind");
    // membership bits: bit e of word e/32 is, on this little-endian host, bit (e % 8) of byte e/8
    std::vector<uint8_t> bits(((size_t)G.m + 7) / 8, 0);
    if (G.m) CGB_CUDA(cudaMemcpyAsync(bits.data(), C.fbits.get(), bits.size(), cudaMemcpyDeviceToHost, s));
    const unsigned long long h = graph_hash(G, s);  // (synchronises s)
    CoreFileHeader hd{};
    std::memcpy(hd.magic, kMagic, 8);
    hd.version = 1;
    hd.kind = (uint32_t)kind;
    hd.alg = (uint32_t)C.alg;
    hd.connectivity = (uint32_t)C.connectivity;
    hd.K = (uint32_t)C.hubs.size();
    hd.n = G.n;
    hd.m = G.m;
    hd.graph_hash = h;
    hd.m_cg = C.m_cg;
    FILE* fp = std::fopen(path, "wb");
    CGB_CHECK(fp != nullptr, CG_EINVAL, std::string("cannot open for writing: ") + path);
    bool ok = std::fwrite(&hd, sizeof hd, 1, fp) == 1;
    ok = ok && (C.hubs.empty() || std::fwrite(C.hubs.data(), 4, C.hubs.size(), fp) == C.hubs.size());
    ok = ok && (bits.empty() || std::fwrite(bits.data(), 1, bits.size(), fp) == bits.size());
    ok = (std::fclose(fp) == 0) && ok;
    CGB_CHECK(ok, CG_EINVAL, std::string("write failed: ") + path);
}

void load_core(Graph& G, int kind, const char* path, cudaStream_t s) {
    FILE* fp = std::fopen(path, "rb");
    CGB_CHECK(fp != nullptr, CG_EINVAL, std::string("cannot open: ") + path);
    CoreFileHeader hd{};
    bool ok = std::fread(&hd, sizeof hd, 1, fp) == 1 && std::memcmp(hd.magic, kMagic, 8) == 0 && hd.version == 1;
    std::vector<uint32_t> hubs(ok ? hd.K : 0);
    std::vector<uint8_t> bits(ok ? ((size_t)hd.m + 7) / 8 : 0);
    ok = ok && (hubs.empty() || std::fread(hubs.data(), 4, hubs.size(), fp) == hubs.size());
    ok = ok && (bits.empty() || std::fread(bits.data(), 1, bits.size(), fp) == bits.size());
    std::fclose(fp);
    CGB_CHECK(ok, CG_EINVAL, std::string("not a Core Graph file (or truncated): ") + path);
    CGB_CHECK((int)hd.kind == kind || core_slot((int)hd.kind) == core_slot(kind), CG_EINVAL,
              "the file holds the Core Graph of another kind");
    CGB_CHECK(hd.n == G.n && hd.m == G.m && hd.graph_hash == graph_hash(G, s), CG_EINVAL,
              "the file was saved for another graph (n, m or fingerprint differ)");
    if (G.m % 8) bits.back() &= (uint8_t)((1u << (G.m % 8)) - 1u);  // no stray bits past edge m-1
    Timer t(s);
    Core& C = G.core[core_slot(kind)];
    C.built = false;
    C.sym_built = false;
    C.hub_vals.reset();
    C.hub_k = 0;
    C.fbits.alloc(((size_t)G.m + 31) / 32 + 1, s);
    CGB_CUDA(cudaMemsetAsync(C.fbits.get(), 0, C.fbits.bytes(), s));
    if (G.m) CGB_CUDA(cudaMemcpyAsync(C.fbits.get(), bits.data(), bits.size(), cudaMemcpyHostToDevice, s));
    split_core(G, C, s);  // the saved bits already hold the connectivity edges
    CGB_CHECK(C.m_cg == hd.m_cg, CG_EINVAL, "Core Graph file is inconsistent (edge count)");
    C.hubs = hubs;
    C.alg = (int)hd.alg;
    C.connectivity = (int)hd.connectivity;
    C.build_ms = t.stop();
    C.built = true;
}

void export_core_flags(Graph& G, const Core& C, uint8_t* flags, cudaStream_t s) {
    if (G.m) CGB_LAUNCH(k_unpack_bits, 4 * G.num_sms, TB, 0, s, (uint64_t)G.m, C.fbits.get(), flags);
}

}  // namespace cgb
