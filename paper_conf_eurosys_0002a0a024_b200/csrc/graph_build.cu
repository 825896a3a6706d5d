// graph_build.cu — canonical CSR / CSC builder.
//
// G(V,E) is canonicalised per reading Q14: self-loops dropped,
// parallel edges collapsed to the minimum weight, rows sorted by destination.  G^R
// (Alg 1 l.5 P:741, Alg 2 l.7 P:1043) is stored as a CSR of the reversed edges with a
// map back to G's edge positions (needed by Alg 2's Reverse(E_b)).
//
// Pipeline (all on device): validate -> key (src<<32|dst) -> radix sort pairs (CUB,
// library call in the one-time builder) -> run heads + min weight -> scan -> scatter ->
// row offsets -> packed edge words; then the same for (dst<<32|src) to get G^R.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "graph.hpp"

namespace cgb {

namespace {

constexpr int TB = 256;

inline int grid_for(uint64_t items, int tb = TB) {
    uint64_t g = (items + tb - 1) / tb;
    if (g > (1u << 20)) g = 1u << 20;
    return (int)(g ? g : 1);
}

inline uint32_t bitlen(uint64_t x) {
    uint32_t b = 0;
    while (x) { ++b; x >>= 1; }
    return b;
}

__global__ void k_validate(uint64_t m, uint32_t n, const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst,
                           const uint32_t* __restrict__ w, uint32_t* flags /* [0]=bad id [1]=bad w [2]=w_max */) {
    uint32_t wmax = 0, bad_id = 0, bad_w = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t a = src[i], b = dst[i], c = w[i];
        bad_id |= (a >= n) | (b >= n);
        bad_w |= (c == 0);
        if (a != b && c > wmax) wmax = c;  // self-loops are dropped, their weight does not count
    }
    if (bad_id) atomicOr(&flags[0], 1u);
    if (bad_w) atomicOr(&flags[1], 1u);
    for (int o = 16; o > 0; o >>= 1) wmax = max(wmax, __shfl_xor_sync(0xffffffffu, wmax, o));
    if ((threadIdx.x & 31) == 0 && wmax) atomicMax(&flags[2], wmax);
}

__global__ void k_make_keys(uint64_t m, uint64_t sentinel, const uint32_t* __restrict__ a, const uint32_t* __restrict__ b,
                            const uint32_t* __restrict__ w, unsigned long long* __restrict__ keys,
                            uint32_t* __restrict__ vals) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t u = a[i], v = b[i];
        keys[i] = (u == v) ? sentinel : (((unsigned long long)u << 32) | v);
        vals[i] = w[i];
    }
}

// head[i] = 1 iff key[i] starts a run of equal valid keys
__global__ void k_heads(uint64_t m, uint64_t sentinel, const unsigned long long* __restrict__ keys,
                        uint32_t* __restrict__ head) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long k = keys[i];
        head[i] = (k < sentinel) && (i == 0 || keys[i - 1] != k);
    }
}

// canonical edge pos[i] <- run starting at i, weight = min over the run
__global__ void k_scatter_runs(uint64_t m, const unsigned long long* __restrict__ keys, const uint32_t* __restrict__ vals,
                               const uint32_t* __restrict__ head, const uint32_t* __restrict__ pos,
                               uint32_t* __restrict__ csrc, uint32_t* __restrict__ cdst, uint32_t* __restrict__ cw) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        if (!head[i]) continue;
        unsigned long long k = keys[i];
        uint32_t wm = vals[i];
        for (uint64_t j = i + 1; j < m && keys[j] == k; ++j) wm = min(wm, vals[j]);
        uint32_t p = pos[i];
        csrc[p] = (uint32_t)(k >> 32);
        cdst[p] = (uint32_t)k;
        cw[p] = wm;
    }
}

// row offsets from a source-sorted edge array: ptr[u] = first edge with src >= u
__global__ void k_row_ptr(uint32_t mc, uint32_t n, const uint32_t* __restrict__ esrc, uint32_t* __restrict__ ptr) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i <= mc; i += (uint64_t)gridDim.x * blockDim.x) {
        int64_t cur = (i < mc) ? (int64_t)esrc[i] : (int64_t)n;  // virtual edge mc has source n
        int64_t prev = (i == 0) ? -1 : (int64_t)esrc[i - 1];
        for (int64_t u = prev + 1; u <= cur; ++u) ptr[u] = (uint32_t)i;
    }
}

__global__ void k_pack(uint32_t m, uint32_t dbits, int packed, const uint32_t* __restrict__ idx,
                       const uint32_t* __restrict__ w, const uint32_t* __restrict__ perm, uint32_t* __restrict__ adj,
                       uint2* __restrict__ adjw) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t wi = perm ? w[perm[i]] : w[i];
        if (packed) adj[i] = idx[i] | ((wi - 1u) << dbits);
        else adjw[i] = make_uint2(idx[i], wi);
    }
}

__global__ void k_rev_keys(uint32_t m, const uint32_t* __restrict__ csrc, const uint32_t* __restrict__ cdst,
                           unsigned long long* __restrict__ keys, uint32_t* __restrict__ vals) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        keys[i] = ((unsigned long long)cdst[i] << 32) | csrc[i];
        vals[i] = (uint32_t)i;
    }
}

__global__ void k_split_keys(uint32_t m, const unsigned long long* __restrict__ keys, uint32_t* __restrict__ hi,
                             uint32_t* __restrict__ lo) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        hi[i] = (uint32_t)(keys[i] >> 32);
        lo[i] = (uint32_t)keys[i];
    }
}

__global__ void k_export(uint32_t n, uint32_t m, uint32_t dbits, const uint32_t* __restrict__ ptr32,
                         const uint32_t* __restrict__ adj, const uint2* __restrict__ adjw, int64_t* __restrict__ ptr,
                         uint32_t* __restrict__ idx, uint32_t* __restrict__ w) {
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    for (uint64_t i = t; i <= n; i += stride) ptr[i] = ptr32[i];
    uint32_t mask = dbits >= 32 ? 0xffffffffu : ((1u << dbits) - 1u);
    for (uint64_t i = t; idx && i < m; i += stride) {
        uint32_t d, ww;
        if (adj) { uint32_t x = adj[i]; d = x & mask; ww = (x >> dbits) + 1u; }
        else { uint2 x = adjw[i]; d = x.x; ww = x.y; }
        idx[i] = d;
        w[i] = ww;
    }
}

template <typename KeyT, typename ValT>
void radix_sort_pairs(const KeyT* kin, KeyT* kout, const ValT* vin, ValT* vout, uint64_t m, int end_bit,
                      cudaStream_t s) {
    size_t tmp = 0;
    CGB_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp, kin, kout, vin, vout, (int64_t)m, 0, end_bit, s));
    DevBuf<uint8_t> t(tmp, s);
    CGB_CUDA(cub::DeviceRadixSort::SortPairs(t.get(), tmp, kin, kout, vin, vout, (int64_t)m, 0, end_bit, s));
    count_launch(2 * ((end_bit + 7) / 8) + 2);
}

void exclusive_sum(const uint32_t* in, uint32_t* out, uint64_t m, cudaStream_t s) {
    size_t tmp = 0;
    CGB_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, in, out, (int64_t)m, s));
    DevBuf<uint8_t> t(tmp, s);
    CGB_CUDA(cub::DeviceScan::ExclusiveSum(t.get(), tmp, in, out, (int64_t)m, s));
    count_launch(2);
}

}  // namespace

void build_graph(Graph& G, int64_t n64, int64_t m64, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                 cudaStream_t s) {
    CGB_CHECK(n64 > 0, CG_EINVAL, "n must be > 0");
    CGB_CHECK(m64 >= 0, CG_EINVAL, "m must be >= 0");
    CGB_CHECK(n64 < 0xFFFFFFFFll, CG_EOVERFLOW, "n must be < 2^32-1");
    CGB_CHECK(m64 < 0xFFFFFFFFll, CG_EOVERFLOW, "m must be < 2^32-1 (u32 edge offsets)");
    CGB_CHECK(m64 == 0 || (src && dst && w), CG_EINVAL, "null edge array");
    const uint32_t n = (uint32_t)n64;
    const uint64_t m = (uint64_t)m64;
    G.n = n;

    // 1. validate, w_max
    DevBuf<uint32_t> flags(3, s);
    CGB_CUDA(cudaMemsetAsync(flags.get(), 0, 3 * sizeof(uint32_t), s));
    if (m) CGB_LAUNCH(k_validate, grid_for(m), TB, 0, s, m, n, src, dst, w, flags.get());
    uint32_t hf[3];
    CGB_CUDA(cudaMemcpyAsync(hf, flags.get(), sizeof hf, cudaMemcpyDeviceToHost, s));
    CGB_CUDA(cudaStreamSynchronize(s));
    CGB_CHECK(!hf[0], CG_EINVAL, "vertex id >= n in the edge list");
    CGB_CHECK(!hf[1], CG_EINVAL, "edge weight 0 (weights must be >= 1)");
    G.w_max = hf[2] ? hf[2] : 1;
    G.dbits = bitlen(n > 1 ? n - 1 : 1);
    G.packed = G.dbits < 32 && (uint64_t)(G.w_max - 1) < (1ull << (32 - G.dbits));

    // 2. sort (src, dst) keys with weights, self-loops to the end
    const uint64_t sentinel = (uint64_t)n << 32;
    const int end_bit = 32 + (int)bitlen(n);
    uint32_t mc = 0;
    DevBuf<uint32_t> csrc, cdst, cw;
    {
        DevBuf<unsigned long long> k0(m ? m : 1, s), k1(m ? m : 1, s);
        DevBuf<uint32_t> v0(m ? m : 1, s), v1(m ? m : 1, s);
        if (m) {
            CGB_LAUNCH(k_make_keys, grid_for(m), TB, 0, s, m, sentinel, src, dst, w, k0.get(), v0.get());
            radix_sort_pairs(k0.get(), k1.get(), v0.get(), v1.get(), m, end_bit, s);
            // 3. run heads, positions (reuse k0/v0 storage)
            uint32_t* head = v0.get();
            DevBuf<uint32_t> pos(m, s);
            CGB_LAUNCH(k_heads, grid_for(m), TB, 0, s, m, sentinel, k1.get(), head);
            exclusive_sum(head, pos.get(), m, s);
            uint32_t last_pos = 0, last_head = 0;
            CGB_CUDA(cudaMemcpyAsync(&last_pos, pos.get() + (m - 1), 4, cudaMemcpyDeviceToHost, s));
            CGB_CUDA(cudaMemcpyAsync(&last_head, head + (m - 1), 4, cudaMemcpyDeviceToHost, s));
            CGB_CUDA(cudaStreamSynchronize(s));
            mc = last_pos + last_head;
            csrc.alloc(mc ? mc : 1, s);
            cdst.alloc(mc ? mc : 1, s);
            cw.alloc(mc ? mc : 1, s);
            CGB_LAUNCH(k_scatter_runs, grid_for(m), TB, 0, s, m, k1.get(), v1.get(), head, pos.get(), csrc.get(),
                       cdst.get(), cw.get());
        }
    }
    G.m = mc;
    G.g.n = G.gr.n = n;
    G.g.m = G.gr.m = mc;

    // 4. CSR of G
    G.g.ptr.alloc(n + 1, s);
    CGB_LAUNCH(k_row_ptr, grid_for((uint64_t)mc + 1), TB, 0, s, mc, n, csrc.get(), G.g.ptr.get());
    if (G.packed) G.g.adj.alloc(adj_alloc_elems(mc, 4), s); else G.g.adjw.alloc(adj_alloc_elems(mc, 8), s);
    if (mc)
        CGB_LAUNCH(k_pack, grid_for(mc), TB, 0, s, mc, G.dbits, (int)G.packed, cdst.get(), cw.get(),
                   (const uint32_t*)nullptr, G.g.adj.get(), G.g.adjw.get());

    // 5. G^R: sort (dst, src) with the CSR edge index as value
    G.gr.ptr.alloc(n + 1, s);
    G.reid.alloc(mc ? mc : 1, s);
    if (G.packed) G.gr.adj.alloc(adj_alloc_elems(mc, 4), s); else G.gr.adjw.alloc(adj_alloc_elems(mc, 8), s);
    {
        DevBuf<uint32_t> rsrc(mc ? mc : 1, s), rrow(mc ? mc : 1, s);
        if (mc) {
            DevBuf<unsigned long long> k0(mc, s), k1(mc, s);
            DevBuf<uint32_t> v0(mc, s);
            CGB_LAUNCH(k_rev_keys, grid_for(mc), TB, 0, s, mc, csrc.get(), cdst.get(), k0.get(), v0.get());
            radix_sort_pairs(k0.get(), k1.get(), v0.get(), G.reid.get(), mc, 32 + (int)bitlen(n), s);
            CGB_LAUNCH(k_split_keys, grid_for(mc), TB, 0, s, mc, k1.get(), rsrc.get(), rrow.get());
        }
        CGB_LAUNCH(k_row_ptr, grid_for((uint64_t)mc + 1), TB, 0, s, mc, n, rsrc.get(), G.gr.ptr.get());
        if (mc)
            CGB_LAUNCH(k_pack, grid_for(mc), TB, 0, s, mc, G.dbits, (int)G.packed, rrow.get(), cw.get(),
                       G.reid.get(), G.gr.adj.get(), G.gr.adjw.get());
    }
    CGB_CUDA(cudaStreamSynchronize(s));
}

void export_adj(const Graph& G, const Adj& a, int64_t* ptr, uint32_t* idx, uint32_t* w, cudaStream_t s) {
    CGB_LAUNCH(k_export, grid_for((uint64_t)a.m + a.n + 1), TB, 0, s, a.n, a.m, G.dbits, a.ptr.get(), a.adj.get(),
               a.adjw.get(), ptr, idx, w);
}

}  // namespace cgb
