// kernels.cuh — device building blocks shared by the query engines (engine.cu: one query per
// pass; engine_batch.cu: a batch of sources per pass).  Internal, not part of the ABI.
#pragma once

#include "graph.hpp"

namespace cgb {
namespace kern {

constexpr uint32_t FULL = 0xffffffffu;
constexpr int CW = 8;  // bitmap words whose degrees are fetched at once in S1

// ------------------------------------------------------------------ kinds (Table 6)
template <int KIND> struct Op;
template <> struct Op<CG_SSSP> {
    static constexpr uint32_t INIT = 0xffffffffu, SRC = 0u;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) { return a + w; }
    __device__ static bool better(uint32_t a, uint32_t b) { return a < b; }
    __device__ static void edge_fn(uint32_t* p, uint32_t v) { red_min(p, v); }
};
template <> struct Op<CG_SSWP> {
    static constexpr uint32_t INIT = 0u, SRC = 0xffffffffu;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) { return min(a, w); }
    __device__ static bool better(uint32_t a, uint32_t b) { return a > b; }
    __device__ static void edge_fn(uint32_t* p, uint32_t v) { red_max(p, v); }
};
template <> struct Op<CG_SSNP> {
    static constexpr uint32_t INIT = 0xffffffffu, SRC = 0u;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) { return max(a, w); }
    __device__ static bool better(uint32_t a, uint32_t b) { return a < b; }
    __device__ static void edge_fn(uint32_t* p, uint32_t v) { red_min(p, v); }
};
// Viterbi: binary32 probabilities in [0,1]; for non-negative floats the u32 bit pattern
// orders exactly like the value, so CASMAX is red.max.u32 on the bits (no CAS loop).
template <> struct Op<CG_VITERBI> {
    static constexpr uint32_t INIT = 0x00000000u /* 0.0f */, SRC = 0x3f800000u /* 1.0f */;
    __device__ static uint32_t ext(uint32_t a, uint32_t w) {
        return __float_as_uint(__fdiv_rn(__uint_as_float(a), __uint2float_rn(w)));
    }
    __device__ static bool better(uint32_t a, uint32_t b) { return a > b; }
    __device__ static void edge_fn(uint32_t* p, uint32_t v) { red_max(p, v); }
};
// Viterbi's Val(u)/w rounded to nearest (reading Q13), with the per-edge reciprocal hoisted out
// of a batch row: for w <= 64 and x = Val(u) >= 2^-64, r = RN(1/w) once per edge, q = RN(x*r),
// the residual e = x - q*w exactly (one FMA), and Markstein's correction RN(q + e*r) — equal
// to RN(x/w) for every such x and w.  tests/test_viterbi_div.py checks that exhaustively (all
// 2^23 significands of three binades x every w <= 64); within the fast range neither the
// quotient nor the residual leaves the normal range, so each result scales exactly with x's
// exponent and the three binades cover it.  Otherwise: __fdiv_rn.
struct VitArg {
    uint32_t w;
    float r;  // RN(1/w), or 0 (slow path)
};
// (the batched engine builds it as {w, w <= 64 ? RN(1/w) : 0} from a per-CTA table, engine_batch.cu s_rcp)
__device__ __forceinline__ uint32_t vit_div(uint32_t a, const VitArg& A) {
    const float x = __uint_as_float(a);
    const float b = __uint2float_rn(A.w);  // exact for w <= 64
    const float q = __fmul_rn(x, A.r);
    const float e = __fmaf_rn(-q, b, x);
    float y = __fmaf_rn(e, A.r, q);
    if (!(A.r != 0.0f && x >= 0x1p-64f)) y = __fdiv_rn(x, b);  // rare: large w or a tiny value
    return __float_as_uint(y);
}

// the N quotients of one edge (a batch row's relax group): the fast path for all N, one
// warp-divergent branch to __fdiv_rn only when some lane falls outside it
template <int N>
__device__ __forceinline__ void vit_div4(const uint32_t (&a)[N], const VitArg& A, uint32_t (&out)[N]) {
    const float b = __uint2float_rn(A.w);
    // a lane leaves the fast path iff 0 < x < 2^-64 (0 / w = 0 on the fast path too); values are
    // non-negative binary32, whose bit patterns order like the values and 2^-64 is 0x1F800000, so
    // that is (bits - 1) < 0x1F7FFFFF unsigned: one min per lane instead of two compares
    uint32_t lo = 0xffffffffu;
#pragma unroll
    for (int i = 0; i < N; ++i) {
        const float x = __uint_as_float(a[i]);
        const float q = __fmul_rn(x, A.r);
        const float e = __fmaf_rn(-q, b, x);
        out[i] = __float_as_uint(__fmaf_rn(e, A.r, q));
        lo = min(lo, a[i] - 1u);
    }
    const bool slow = A.r == 0.0f || lo < 0x1F7FFFFFu;
    if (slow) {
#pragma unroll
        for (int i = 0; i < N; ++i) out[i] = vit_div(a[i], A);
    }
}

template <> struct Op<CG_BFS> {
    static constexpr uint32_t INIT = 0xffffffffu, SRC = 0u;
    __device__ static uint32_t ext(uint32_t a, uint32_t) { return a + 1u; }
    __device__ static bool better(uint32_t a, uint32_t b) { return a < b; }
    __device__ static void edge_fn(uint32_t* p, uint32_t v) { red_min(p, v); }
};
template <> struct Op<CG_REACH> {
    static constexpr uint32_t INIT = 0u, SRC = 1u;
    __device__ static uint32_t ext(uint32_t a, uint32_t) { return a; }
    __device__ static bool better(uint32_t a, uint32_t b) { return a > b; }
    __device__ static void edge_fn(uint32_t* p, uint32_t v) { red_max(p, v); }
};

// the graph's sticky error word lives in host-mapped pinned memory (read by the next API call
// on the graph, or by cg_graph_status after a stream sync); only thread 0 of the grid writes it
__device__ __forceinline__ void report_sticky(uint32_t* err_map, uint32_t e) {
    if (!e || !err_map) return;
    volatile uint32_t* p = err_map;
    *p = *p | e;
    __threadfence_system();
}

// ------------------------------------------------------------------ grid barrier
#ifndef CGB_BAR_SLEEP
#define CGB_BAR_SLEEP 32  // ns between polls of the arrival counter (0: spin)
#endif
__device__ __forceinline__ void grid_sync(unsigned long long* bar, unsigned long long& epoch) {
    __syncthreads();
    ++epoch;
    if (threadIdx.x == 0) {
        const unsigned long long target = epoch * gridDim.x;
        asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(bar) : "memory");
        unsigned long long cur;
        for (;;) {  // relaxed polling: no per-poll L1 invalidation
            asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(cur) : "l"(bar) : "memory");
            if (cur >= target) break;
#if CGB_BAR_SLEEP
            __nanosleep(CGB_BAR_SLEEP);
#endif
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
    }
    __syncthreads();
}

__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

template <int NWARPS, typename T>
__device__ __forceinline__ T block_sum(T v, T* sm /* NWARPS */) {
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = v;
    __syncthreads();
    T t = 0;
    if (threadIdx.x < 32) {
        t = threadIdx.x < NWARPS ? sm[threadIdx.x] : 0;
        for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(FULL, t, o);
    }
    return t;  // valid in thread 0
}

// ------------------------------------------------------------------ edge access
template <bool PACKED>
struct EdgeWord;
template <>
struct EdgeWord<true> {
    uint32_t x;
    __device__ void load(const GraphView& g, uint32_t e) { x = ld_stream(g.adj + e); }
    __device__ void decode(uint32_t dbits, uint32_t dmask, uint32_t& d, uint32_t& w) const {
        d = x & dmask;
        w = (x >> dbits) + 1u;
    }
};
template <>
struct EdgeWord<false> {
    uint2 x;
    __device__ void load(const GraphView& g, uint32_t e) { x = ld_stream2(g.adjw + e); }
    __device__ void decode(uint32_t, uint32_t, uint32_t& d, uint32_t& w) const {
        d = x.x;
        w = x.y;
    }
};

// Degrees of the 32 vertices of up to CW nonzero bitmap words taken from `nz` (lane = vertex:
// one coalesced 128 B row-offset read per word; lane 31 fetches the next offset; split rows
// read their row ends too).
__device__ __forceinline__ void word_degrees(const GraphView& g, uint32_t n, uint32_t g0, uint32_t& nz, uint32_t lane,
                                             int (&js)[CW], uint32_t (&deg)[CW]) {
    uint32_t p0[CW], p1[CW];
#pragma unroll
    for (int k = 0; k < CW; ++k) {
        js[k] = -1;
        if (nz) {
            js[k] = __ffs(nz) - 1;
            nz &= nz - 1;
        }
    }
    if (g.end) {  // split rows: [ptr[v], end[v]) (vertices past n have no row: v < n checked)
#pragma unroll
        for (int k = 0; k < CW; ++k) {
            p0[k] = p1[k] = 0;
            const uint32_t v = (g0 + js[k]) * 32 + lane;
            if (js[k] >= 0 && v < n) {
                p0[k] = __ldg(g.ptr + v);
                p1[k] = __ldg(g.end + v);
            }
        }
#pragma unroll
        for (int k = 0; k < CW; ++k) deg[k] = p1[k] - p0[k];
        return;
    }
#pragma unroll
    for (int k = 0; k < CW; ++k) {
        p0[k] = p1[k] = 0;
        if (js[k] >= 0) {
            const uint32_t v = min((g0 + js[k]) * 32 + lane, n);
            p0[k] = __ldg(g.ptr + v);
            if (lane == 31) p1[k] = __ldg(g.ptr + min(v + 1, n));
        }
    }
#pragma unroll
    for (int k = 0; k < CW; ++k) {
        uint32_t nx = __shfl_down_sync(FULL, p0[k], 1);
        if (lane == 31) nx = p1[k];
        deg[k] = nx - p0[k];
    }
}

}  // namespace kern
}  // namespace cgb
