// Microbenchmark (not part of the library): achievable HBM bandwidth of kernel A's access
// pattern on this B200 — each warp gathers k random 2 KB chunks (16 B per lane x 4) of
// rows in a large array and writes one 2 KB chunk sequentially — against a plain copy.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_bw gather_bw.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256, 4) gather(const uint4* __restrict__ src, uint4* __restrict__ dst,
                                                 const uint32_t* __restrict__ rows, uint32_t nwarps,
                                                 uint32_t row_vec, int k) {
    const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    if (w >= nwarps) return;
    const uint32_t cpg = row_vec / 128;                 // 4 vectors per lane per chunk
    const uint32_t gate = w / cpg, chunk = w % cpg;
    uint4 x[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        if (i >= k) break;
        const uint4* s = src + (uint64_t)__ldg(rows + gate * 4 + i) * row_vec + chunk * 128 + lane;
#pragma unroll
        for (int u = 0; u < 4; ++u) x[u][i] = __ldg(s + u * 32);
    }
    uint4* d = dst + (uint64_t)gate * row_vec + chunk * 128 + lane;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        uint4 y = x[u][0];
        for (int i = 1; i < k; ++i) { y.x ^= x[u][i].x; y.y &= x[u][i].y; y.z |= x[u][i].z; y.w ^= x[u][i].w; }
        d[u * 32] = y;
    }
}

__global__ void copyk(const uint4* __restrict__ s, uint4* __restrict__ d, uint64_t n) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        d[i] = __ldg(s + i);
}

int main() {
    const uint64_t row_bytes = 8192, nrows = 1u << 20;           // 8 GiB of rows (C4-like)
    const uint64_t row_vec = row_bytes / 16;
    uint4 *src, *dst;
    cudaMalloc(&src, nrows * row_bytes);
    cudaMalloc(&dst, 16384ull * row_bytes);
    cudaMemset(src, 1, nrows * row_bytes);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int k : {1, 2, 3, 4}) {
        const uint32_t ngates = 14500;
        std::vector<uint32_t> h(ngates * 4);
        uint64_t x = 88172645463325252ull;
        for (auto& r : h) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; r = (uint32_t)(x % nrows); }
        uint32_t* rows;
        cudaMalloc(&rows, h.size() * 4);
        cudaMemcpy(rows, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
        const uint32_t nwarps = ngates * (row_vec / 128);
        for (int it = 0; it < 3; ++it) gather<<<(nwarps * 32 + 255) / 256, 256>>>(src, dst, rows, nwarps, row_vec, k);
        cudaEventRecord(a);
        const int reps = 20;
        for (int it = 0; it < reps; ++it) gather<<<(nwarps * 32 + 255) / 256, 256>>>(src, dst, rows, nwarps, row_vec, k);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        const double bytes = (double)ngates * row_bytes * (k + 1) * reps;
        printf("gather k=%d: %.1f GB/s (%.1f us per launch)\n", k, bytes / (ms / 1e3) / 1e9, ms * 1e3 / reps);
        cudaFree(rows);
    }
    const uint64_t n = 2ull * 1024 * 1024 * 1024 / 16;     // 2 GiB copy
    for (int it = 0; it < 3; ++it) copyk<<<148 * 8, 256>>>(src, dst == nullptr ? nullptr : src + n, n);
    cudaEventRecord(a);
    for (int it = 0; it < 10; ++it) copyk<<<148 * 8, 256>>>(src, src + n, n);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("copy: %.1f GB/s\n", 2.0 * n * 16 * 10 / (ms / 1e3) / 1e9);
    return 0;
}
