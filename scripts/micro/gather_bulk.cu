// Microbenchmark (not part of the library): does staging kernel A's gathers through the bulk
// copy engine (cp.async.bulk global->shared, mbarrier completion, S-stage ring per CTA) beat
// the register gather (16 B per lane, 4 vectors in flight) on this B200?  Each item = one
// gate x one C-byte chunk of its rows: k random input chunks in, one sequential chunk out.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_bulk gather_bulk.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
                     : "=r"(done) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    }
}

template <int C, int S>
__global__ void __launch_bounds__(256) gather_bulk(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                                   const uint32_t* __restrict__ rows, uint32_t nitems,
                                                   uint32_t row_bytes, int k) {
    extern __shared__ __align__(128) uint8_t sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm);
    uint8_t* buf = sm + 128;
    const uint32_t cpg = row_bytes / C;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) mbar_init(&full[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](uint32_t j, int s) {
        const uint32_t item = blockIdx.x + j * gridDim.x;
        if (item >= nitems) return;
        const uint32_t gate = item / cpg, chunk = item % cpg;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect(&full[s], C * k);
        for (int i = 0; i < k; ++i)
            bulk_load(buf + (s * 4 + i) * C, src + (uint64_t)rows[gate * 4 + i] * row_bytes + (uint64_t)chunk * C, C,
                      &full[s]);
    };
    if (threadIdx.x == 0)
        for (int s = 0; s < S; ++s) issue(s, s);
    for (uint32_t j = 0;; ++j) {
        const uint32_t item = blockIdx.x + j * gridDim.x;
        if (item >= nitems) break;
        const int s = j % S;
        mbar_wait(&full[s], (j / S) & 1);
        const uint32_t gate = item / cpg, chunk = item % cpg;
        const uint4* x = reinterpret_cast<const uint4*>(buf + s * 4 * C);
        uint4* d = reinterpret_cast<uint4*>(dst + (uint64_t)gate * row_bytes + (uint64_t)chunk * C);
#pragma unroll
        for (int v = threadIdx.x; v < C / 16; v += 256) {
            uint4 y = x[v];
            for (int i = 1; i < k; ++i) {
                const uint4 z = x[i * (C / 16) + v];
                y.x ^= z.x; y.y &= z.y; y.z |= z.z; y.w ^= z.w;
            }
            d[v] = y;
        }
        __syncthreads();
        if (threadIdx.x == 0) issue(j + S, s);
    }
}

// The register gather of kernel A's wide path (U vectors of 16 B per lane per input row).
template <int U>
__global__ void __launch_bounds__(256) gather_reg(const uint4* __restrict__ src, uint4* __restrict__ dst,
                                                  const uint32_t* __restrict__ rows, uint32_t nwarps,
                                                  uint32_t row_vec, int k) {
    const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    if (w >= nwarps) return;
    const uint32_t cpg = row_vec / (32 * U);
    const uint32_t gate = w / cpg, chunk = w % cpg;
    uint4 x[U][4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        if (i >= k) break;
        const uint4* s = src + (uint64_t)__ldg(rows + gate * 4 + i) * row_vec + chunk * 32 * U + lane;
#pragma unroll
        for (int u = 0; u < U; ++u) x[u][i] = __ldg(s + u * 32);
    }
    uint4* d = dst + (uint64_t)gate * row_vec + chunk * 32 * U + lane;
#pragma unroll
    for (int u = 0; u < U; ++u) {
        uint4 y = x[u][0];
        for (int i = 1; i < k; ++i) { y.x ^= x[u][i].x; y.y &= x[u][i].y; y.z |= x[u][i].z; y.w ^= x[u][i].w; }
        d[u * 32] = y;
    }
}

__global__ void copyk(const uint4* __restrict__ s, uint4* __restrict__ d, uint64_t n) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        d[i] = __ldg(s + i);
}

static cudaEvent_t ea, eb;
template <typename F>
static double time_it(F f, int reps) {
    for (int i = 0; i < 3; ++i) f();
    cudaEventRecord(ea);
    for (int i = 0; i < reps; ++i) f();
    cudaEventRecord(eb);
    cudaEventSynchronize(eb);
    float ms;
    cudaEventElapsedTime(&ms, ea, eb);
    return ms / reps;
}

template <int C, int S>
static void run_bulk(const uint8_t* src, uint8_t* dst, const uint32_t* rows, uint32_t ngates, uint32_t row_bytes,
                     int k, int ctas_per_sm) {
    const uint32_t nitems = ngates * (row_bytes / C);
    const size_t smem = 128 + (size_t)S * 4 * C;
    cudaFuncSetAttribute(gather_bulk<C, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const uint32_t grid = 148 * ctas_per_sm;
    const double ms = time_it([&] { gather_bulk<C, S><<<grid, 256, smem>>>(src, dst, rows, nitems, row_bytes, k); }, 20);
    cudaError_t e = cudaGetLastError();
    printf("bulk C=%5d S=%d ctas/sm=%d k=%d: %7.1f GB/s (%.1f us) %s\n", C, S, ctas_per_sm, k,
           (double)ngates * row_bytes * (k + 1) / (ms / 1e3) / 1e9, ms * 1e3, e == cudaSuccess ? "" : cudaGetErrorString(e));
}


// Warp-specialised: warp 0 (one lane) produces — it prefetches the next item's row indices,
// waits for the stage to be released, arms the mbarrier and issues the k bulk copies; warps
// 1..8 consume (evaluate + store) and release the stage.
template <int C, int S>
__global__ void __launch_bounds__(288) gather_ws(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                                 const uint32_t* __restrict__ rows, uint32_t nitems,
                                                 uint32_t row_bytes, int k) {
    extern __shared__ __align__(128) uint8_t sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm);
    uint64_t* empty = full + S;
    uint8_t* buf = sm + 1024;
    const uint32_t cpg = row_bytes / C;
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 8); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (warp == 0) {
        if (lane != 0) return;
        uint32_t item = blockIdx.x;
        uint4 r = item < nitems ? *reinterpret_cast<const uint4*>(rows + (item / cpg) * 4) : make_uint4(0, 0, 0, 0);
        for (uint32_t j = 0; item < nitems; ++j) {
            const uint32_t nxt = item + gridDim.x;
            const uint4 rn = nxt < nitems ? *reinterpret_cast<const uint4*>(rows + (nxt / cpg) * 4) : r;
            const int s = j % S;
            if (j >= S) mbar_wait(&empty[s], ((j / S) - 1) & 1);
            const uint64_t off = (uint64_t)(item % cpg) * C;
            mbar_expect(&full[s], C * k);
            const uint32_t rr[4] = {r.x, r.y, r.z, r.w};
            for (int i = 0; i < k; ++i) bulk_load(buf + (s * 4 + i) * C, src + (uint64_t)rr[i] * row_bytes + off, C, &full[s]);
            item = nxt;
            r = rn;
        }
        return;
    }
    const uint32_t t = threadIdx.x - 32;
    for (uint32_t j = 0;; ++j) {
        const uint32_t item = blockIdx.x + j * gridDim.x;
        if (item >= nitems) break;
        const int s = j % S;
        mbar_wait(&full[s], (j / S) & 1);
        const uint32_t gate = item / cpg, chunk = item % cpg;
        const uint4* x = reinterpret_cast<const uint4*>(buf + s * 4 * C);
        uint4* d = reinterpret_cast<uint4*>(dst + (uint64_t)gate * row_bytes + (uint64_t)chunk * C);
#pragma unroll
        for (int v = t; v < C / 16; v += 256) {
            uint4 y = x[v];
            for (int i = 1; i < k; ++i) {
                const uint4 z = x[i * (C / 16) + v];
                y.x ^= z.x; y.y &= z.y; y.z |= z.z; y.w ^= z.w;
            }
            d[v] = y;
        }
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[s])) : "memory");
    }
}

template <int C, int S>
static void run_ws(const uint8_t* src, uint8_t* dst, const uint32_t* rows, uint32_t ngates, uint32_t row_bytes,
                   int k, int ctas_per_sm) {
    const uint32_t nitems = ngates * (row_bytes / C);
    const size_t smem = 1024 + (size_t)S * 4 * C;
    cudaFuncSetAttribute(gather_ws<C, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const uint32_t grid = 148 * ctas_per_sm;
    const double ms = time_it([&] { gather_ws<C, S><<<grid, 288, smem>>>(src, dst, rows, nitems, row_bytes, k); }, 20);
    cudaError_t e = cudaGetLastError();
    printf("ws   C=%5d S=%d ctas/sm=%d k=%d: %7.1f GB/s (%.1f us) %s\n", C, S, ctas_per_sm, k,
           (double)ngates * row_bytes * (k + 1) / (ms / 1e3) / 1e9, ms * 1e3, e == cudaSuccess ? "" : cudaGetErrorString(e));
}

template <int U>
static void run_reg(const uint8_t* src, uint8_t* dst, const uint32_t* rows, uint32_t ngates, uint32_t row_bytes, int k) {
    const uint32_t row_vec = row_bytes / 16, nwarps = ngates * (row_vec / (32 * U));
    const double ms = time_it([&] {
        gather_reg<U><<<(nwarps * 32 + 255) / 256, 256>>>((const uint4*)src, (uint4*)dst, rows, nwarps, row_vec, k);
    }, 20);
    printf("reg  U=%d k=%d: %7.1f GB/s (%.1f us)\n", U, k, (double)ngates * row_bytes * (k + 1) / (ms / 1e3) / 1e9,
           ms * 1e3);
}

int main() {
    const uint64_t row_bytes = 8192, nrows = 1u << 20;           // 8 GiB of rows (C4-like)
    uint8_t *src, *dst;
    cudaMalloc(&src, nrows * row_bytes);
    cudaMalloc(&dst, 16384ull * row_bytes);
    cudaMemset(src, 1, nrows * row_bytes);
    cudaEventCreate(&ea);
    cudaEventCreate(&eb);
    const uint32_t ngates = 14500;
    std::vector<uint32_t> h(ngates * 4);
    uint64_t x = 88172645463325252ull;
    for (auto& r : h) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; r = (uint32_t)(x % nrows); }
    uint32_t* rows;
    cudaMalloc(&rows, h.size() * 4);
    cudaMemcpy(rows, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    for (uint64_t rb : {8192ull, 4096ull}) {
      const uint64_t nr = (8ull << 30) / rb;
      const uint32_t ng = (uint32_t)(14500ull * 8192 / rb);
      std::vector<uint32_t> hh(ng * 4);
      for (auto& r : hh) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; r = (uint32_t)(x % nr); }
      uint32_t* rw;
      cudaMalloc(&rw, hh.size() * 4);
      cudaMemcpy(rw, hh.data(), hh.size() * 4, cudaMemcpyHostToDevice);
      printf("--- row bytes %llu\n", (unsigned long long)rb);
      for (int k : {3, 4}) {
        run_reg<4>(src, dst, rw, ng, rb, k);
        run_reg<2>(src, dst, rw, ng, rb, k);
        if (rb == 8192) {
            run_bulk<8192, 3>(src, dst, rw, ng, rb, k, 2);
            run_ws<8192, 2>(src, dst, rw, ng, rb, k, 2);
            run_ws<8192, 3>(src, dst, rw, ng, rb, k, 2);
            run_ws<8192, 6>(src, dst, rw, ng, rb, k, 1);
        }
        run_ws<4096, 3>(src, dst, rw, ng, rb, k, 3);
        run_ws<4096, 4>(src, dst, rw, ng, rb, k, 2);
        run_ws<4096, 8>(src, dst, rw, ng, rb, k, 1);
        run_ws<2048, 6>(src, dst, rw, ng, rb, k, 2);
        run_ws<2048, 12>(src, dst, rw, ng, rb, k, 1);
        run_ws<1024, 12>(src, dst, rw, ng, rb, k, 2);
      }
      cudaFree(rw);
    }
    const uint64_t n = 2ull * 1024 * 1024 * 1024 / 16;
    const double ms = time_it([&] { copyk<<<148 * 8, 256>>>((const uint4*)src, (uint4*)src + n, n); }, 10);
    printf("copy: %.1f GB/s\n", 2.0 * n * 16 / (ms / 1e3) / 1e9);
    return 0;
}
