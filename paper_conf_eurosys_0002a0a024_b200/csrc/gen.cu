// gen.cu — device twin of the seeded R-MAT input generator.
//
// Input synthesis only (no method arithmetic).  The definition lives in gen/rmat.c (host);
// this is an independent device implementation of the same counter-based recipe so
// that large graphs are drawn directly in HBM.  tests/test_gpu_gen.py checks the two
// produce identical edge lists.
#include "graph.hpp"

namespace cgb {

namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

__device__ __forceinline__ uint64_t feistel4(uint64_t x, uint32_t h, const uint64_t* k) {
    const uint64_t mask = (1ull << h) - 1ull;
    uint64_t L = x >> h, R = x & mask;
#pragma unroll
    for (int r = 0; r < 4; ++r) {
        const uint64_t nl = R;
        R = L ^ (mix64(R ^ k[r]) & mask);
        L = nl;
    }
    return (L << h) | R;
}

__global__ void k_rmat(uint64_t n, uint32_t S, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max, uint64_t kL,
                       uint64_t kW, uint64_t k0, uint64_t k1, uint64_t k2, uint64_t k3, int permute, uint64_t e0,
                       uint64_t count, uint32_t* __restrict__ src, uint32_t* __restrict__ dst, uint32_t* __restrict__ w) {
    const uint64_t keys[4] = {k0, k1, k2, k3};
    const uint32_t h = (S + 1) / 2;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t e = e0 + i;
        uint64_t u = 0, v = 0;
        for (uint32_t l = 0; l < S; ++l) {
            const uint32_t x = (uint32_t)(mix64(kL ^ ((e << 6) | l)) >> 32);
            const uint64_t rb = x >= tAB;                       // quadrants (1,0) and (1,1)
            const uint64_t cb = (x >= tA && x < tAB) || x >= tABC;  // quadrants (0,1) and (1,1)
            u |= rb << l;
            v |= cb << l;
        }
        u = (u * n) >> S;
        v = (v * n) >> S;
        if (permute) {
            uint64_t y = feistel4(u, h, keys);
            while (y >= n) y = feistel4(y, h, keys);
            u = y;
            y = feistel4(v, h, keys);
            while (y >= n) y = feistel4(y, h, keys);
            v = y;
        }
        src[i] = (uint32_t)u;
        dst[i] = (uint32_t)v;
        w[i] = 1u + (uint32_t)(mix64(kW ^ e) % (uint64_t)w_max);
    }
}

uint64_t host_mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

}  // namespace

void rmat_generate(uint64_t n, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max, uint64_t seed, int permute,
                   uint64_t e0, uint64_t count, uint32_t* src, uint32_t* dst, uint32_t* w, cudaStream_t s) {
    CGB_CHECK(n > 0 && n < (1ull << 32), CG_EINVAL, "n must be in [1, 2^32)");
    CGB_CHECK(w_max >= 1, CG_EINVAL, "w_max must be >= 1");
    CGB_CHECK(count == 0 || (src && dst && w), CG_EINVAL, "null output");
    if (!count) return;
    uint32_t S = 1;
    while ((1ull << S) < n) ++S;
    const uint64_t kL = host_mix64(seed ^ 0x243F6A8885A308D3ull);
    const uint64_t kW = host_mix64(seed ^ 0xA4093822299F31D0ull);
    uint64_t k[4];
    for (int r = 0; r < 4; ++r) k[r] = host_mix64(seed ^ (0x13198A2E03707344ull + (uint64_t)r));
    uint64_t blocks = (count + 255) / 256;
    if (blocks > 148ull * 64) blocks = 148ull * 64;
    CGB_LAUNCH(k_rmat, (int)blocks, 256, 0, s, n, S, tA, tAB, tABC, w_max, kL, kW, k[0], k[1], k[2], k[3], permute, e0,
               count, src, dst, w);
}

}  // namespace cgb
