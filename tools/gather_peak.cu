// gather_peak.cu — measured ceiling of RANDOM row gathers on this GPU (the access pattern of the
// batched engine's S2: one value row per edge at a data-dependent address).  The HBM "copy" peak in
// MEASURED_PEAKS.json is a sequential-stream figure; this program measures how many random rows per
// second (and DRAM bytes per second) the memory system sustains for row sizes of 4 / 32 / 64 / 128 B
// over a value array the size of C2's (n = 4,847,571 rows), with uniform and with skewed (power-law)
// row indices, and with a plain load or a cp.async (LDGSTS) per 16 B — no compute, maximal occupancy.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_peak tools/gather_peak.cu
//   ./gather_peak [n_rows [index_file]] > profiles/r2_gather_peak.json
// With an index file (uint32 row ids, e.g. the destinations of C2's CSR in edge order, written by
// tools/gather_c2.py) the stream is that file, in file order ("file") and shuffled ("file-shuffled").
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <initializer_list>
#include <utility>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ uint64_t mix(uint64_t x) {
    x += 0x9e3779b97f4a7c15ull;
    x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ull;
    x = (x ^ (x >> 27)) * 0x94d049bb133111ebull;
    return x ^ (x >> 31);
}

// row index of gather i: uniform, or skewed (the product of two uniforms favours small ids; ids are then
// scattered by a multiplicative hash so hot rows are spread over memory like a permuted RMAT graph)
__global__ void make_idx(uint32_t* idx, uint64_t m, uint32_t n, int skew) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t h = mix(i * 2 + 1);
        uint32_t r;
        if (!skew) {
            r = (uint32_t)(((h >> 32) * n) >> 32);
        } else {
            const double u = (double)(h >> 40) / (double)(1ull << 24), v = (double)(mix(h) >> 40) / (double)(1ull << 24);
            const uint32_t k = (uint32_t)(u * u * v * n);  // heavy head
            r = (uint32_t)(((uint64_t)(k * 2654435761u) % n));
        }
        idx[i] = r;
    }
}

// W = 16 B words per row; 4 rows in flight per thread
template <int W>
__global__ void __launch_bounds__(256) gather_ld(const uint4* __restrict__ V, const uint32_t* __restrict__ idx, uint64_t m,
                                                 uint4* sink) {
    uint4 acc = make_uint4(0, 0, 0, 0);
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += 4 * stride) {
        uint4 x[4][W];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t j = i + u * stride;
            const uint32_t r = j < m ? __ldg(idx + j) : 0u;
#pragma unroll
            for (int w = 0; w < W; ++w) x[u][w] = __ldcg(V + (size_t)r * W + w);
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int w = 0; w < W; ++w) acc.x ^= x[u][w].x ^ x[u][w].w, acc.y ^= x[u][w].y ^ x[u][w].z;
    }
    if (acc.x == 0x12345678u) sink[0] = acc;
}

// cooperative: a warp gathers 32 rows per chunk, instruction i moving 16 B piece (lane % W) of row
// i * (32 / W) + lane / W (the batched engine's RowCopy pattern: 32 / W rows per instruction), U chunks
// of 32 rows in flight per warp
template <int W, int U>
__global__ void __launch_bounds__(256) gather_coop(const uint4* __restrict__ V, const uint32_t* __restrict__ idx,
                                                   uint64_t m, uint4* sink) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    uint32_t acc = 0;
    for (uint64_t c = blockIdx.x * (uint64_t)(blockDim.x / 32) + (threadIdx.x >> 5); c * 32 < m; c += U * nw) {
        uint4 x[U][W];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint64_t j = (c + u * nw) * 32 + lane;
            const uint32_t r = j < m ? __ldg(idx + j) : 0u;
#pragma unroll
            for (int i = 0; i < W; ++i) {
                const uint32_t rr = __shfl_sync(0xffffffffu, r, i * (32 / W) + lane / W);
                x[u][i] = __ldcg(V + (size_t)rr * W + lane % W);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int i = 0; i < W; ++i) acc ^= x[u][i].x ^ x[u][i].w;
    }
    if (acc == 0x12345678u) sink[0] = make_uint4(acc, 0, 0, 0);
}

// 4-byte rows
__global__ void __launch_bounds__(256) gather_ld4(const uint32_t* __restrict__ V, const uint32_t* __restrict__ idx,
                                                  uint64_t m, uint32_t* sink) {
    uint32_t acc = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += 8 * stride) {
        uint32_t x[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint64_t j = i + u * stride;
            x[u] = __ldcg(V + (j < m ? __ldg(idx + j) : 0u));
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) acc ^= x[u];
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

// cp.async (LDGSTS) of W x 16 B per row into shared memory, U rows per thread in flight, 128 threads
template <int W, int U>
__global__ void __launch_bounds__(128) gather_cpasync(const uint4* __restrict__ V, const uint32_t* __restrict__ idx,
                                                      uint64_t m, uint4* sink) {
    __shared__ uint4 ring[128 * U * W];
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint32_t acc = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += U * stride) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint64_t j = i + u * stride;
            const uint32_t r = j < m ? __ldg(idx + j) : 0u;
#pragma unroll
            for (int w = 0; w < W; ++w) {
                const uint32_t dst = (uint32_t)__cvta_generic_to_shared(ring + (threadIdx.x * U + u) * W + w);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(V + (size_t)r * W + w) : "memory");
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 0;" ::: "memory");
        acc ^= ring[threadIdx.x * U * W].x;
    }
    if (acc == 0x12345678u) sink[0] = make_uint4(acc, 0, 0, 0);
}

int main(int argc, char** argv) {
    const uint32_t n = argc > 1 ? (uint32_t)atoll(argv[1]) : 4847571u;  // C2's vertex count
    const uint64_t m = 64ull << 20;                                       // gathers per launch
    int dev = 0, sms = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    uint4* V;
    uint32_t* idx;
    uint4* sink;
    CK(cudaMalloc(&V, (size_t)n * 128));
    CK(cudaMemset(V, 1, (size_t)n * 128));
    CK(cudaMalloc(&idx, m * 4));
    CK(cudaMalloc(&sink, 64));
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    std::vector<uint32_t> file;
    if (argc > 2) {
        FILE* f = fopen(argv[2], "rb");
        if (!f) { fprintf(stderr, "cannot open %s\n", argv[2]); return 1; }
        fseek(f, 0, SEEK_END);
        file.resize(ftell(f) / 4);
        fseek(f, 0, SEEK_SET);
        if (fread(file.data(), 4, file.size(), f) != file.size()) return 1;
        fclose(f);
    }
    printf("{\"n_rows\": %u, \"gathers_per_launch\": %llu, \"sms\": %d, \"results\": [\n", n, (unsigned long long)m, sms);
    bool first = true;
    const char* names[4] = {"uniform", "skewed", "file", "file-shuffled"};
    for (int skew = 0; skew < (file.empty() ? 2 : 4); ++skew) {
        if (skew < 2) {
            make_idx<<<sms * 8, 256>>>(idx, m, n, skew);
        } else {  // the file's ids repeated to m gathers; shuffled by a seeded Fisher-Yates for skew 3
            std::vector<uint32_t> h(m);
            for (uint64_t i = 0; i < m; ++i) h[i] = file[i % file.size()] % n;
            if (skew == 3) {
                uint64_t x = 12345;
                for (uint64_t i = m - 1; i > 0; --i) {
                    x = x * 6364136223846793005ull + 1442695040888963407ull;
                    std::swap(h[i], h[(x >> 17) % (i + 1)]);
                }
            }
            CK(cudaMemcpy(idx, h.data(), m * 4, cudaMemcpyHostToDevice));
        }
        CK(cudaDeviceSynchronize());
        for (int kind = 0; kind < 3; ++kind) {
            for (int rb : {4, 32, 64, 128}) {
                if (kind >= 1 && rb == 4) continue;
                const int grid = sms * 8;
                auto launch = [&]() {
                    if (rb == 4) gather_ld4<<<grid, 256>>>(reinterpret_cast<const uint32_t*>(V), idx, m, reinterpret_cast<uint32_t*>(sink));
                    else if (kind == 0 && rb == 32) gather_ld<2><<<grid, 256>>>(V, idx, m, sink);
                    else if (kind == 0 && rb == 64) gather_ld<4><<<grid, 256>>>(V, idx, m, sink);
                    else if (kind == 0 && rb == 128) gather_ld<8><<<grid, 256>>>(V, idx, m, sink);
                    else if (kind == 2 && rb == 32) gather_coop<2, 4><<<grid, 256>>>(V, idx, m, sink);
                    else if (kind == 2 && rb == 64) gather_coop<4, 4><<<grid, 256>>>(V, idx, m, sink);
                    else if (kind == 2 && rb == 128) gather_coop<8, 2><<<grid, 256>>>(V, idx, m, sink);
                    else if (rb == 32) gather_cpasync<2, 4><<<sms * 16, 128>>>(V, idx, m, sink);
                    else if (rb == 64) gather_cpasync<4, 4><<<sms * 6, 128>>>(V, idx, m, sink);
                    else gather_cpasync<8, 2><<<sms * 6, 128>>>(V, idx, m, sink);
                };
                for (int w = 0; w < 3; ++w) launch();
                CK(cudaDeviceSynchronize());
                const int reps = 10;
                CK(cudaEventRecord(a));
                for (int r = 0; r < reps; ++r) launch();
                CK(cudaEventRecord(b));
                CK(cudaEventSynchronize(b));
                CK(cudaGetLastError());
                float ms = 0;
                CK(cudaEventElapsedTime(&ms, a, b));
                const double s = ms / 1e3 / reps;
                printf("%s {\"rows\": \"%s\", \"row_bytes\": %d, \"op\": \"%s\", \"ms\": %.4f, \"G_rows_per_s\": %.2f, "
                       "\"row_GBps\": %.1f}\n",
                       first ? " " : ",", names[skew], rb, kind == 2 ? "ld.global.cg cooperative (32/W rows per instruction)" : kind ? "cp.async.cg" : "ld.global.cg",
                       s * 1e3, m / s / 1e9, m * (double)rb / s / 1e9);
                first = false;
            }
        }
    }
    printf("]}\n");
    return 0;
}
