// kernels.cu — the sm_100a hot path of gsim.
//
// One cycle of the simulated circuit = stimulus rows, then one launch per level
// (the merged NN layers of PAPER.md §III-D), then the end-of-cycle kernel
// (remaining register latches of the recurrent connection P:241, output MISR /
// trace).  State is bit-packed and stimulus-major: row r holds one signal for all
// lanes, 64 stimuli per uint64 word.
//
// Kernel A (k_level_lut): a level is a gather + Boolean evaluation, not a dense
// contraction, so there are no tensor cores here: every thread loads 16 B of each
// input row (coalesced: a warp reads 512 B contiguous per row), evaluates the gate's
// truth table bit-sliced as a Shannon mux tree (2^k - 1 LOP3 per 32 lanes) and
// stores 16 B of the output row (plus the fused latch store into the other Q bank).
//
// Kernel B (k_level_poly): the paper's two-layer network per gate (Fig. 2, P:130;
// Eq. 1-3) evaluated per stimulus in int32: hidden neuron h_S = Theta(sum_{s in S}
// x_s - |S| + 1), output sum_S w_S h_S (only the nonzero w_S, sparse as in P:187),
// then ballot-packed back to 32 stimuli per word.  Outputs outside {0,1} are counted
// (P:224 says they cannot happen).  Used standalone or as a cross-check of A.
#include <algorithm>
#include <atomic>

#include <cuda_runtime.h>

#include "kernels.h"
#include "device.cuh"

namespace gs {

// K = 7, 8 (any vector width VT = uint4 / uint2): the full 256-bit table comes from a.dtt
template <int K, typename VT, typename Args>
__device__ __forceinline__ void lut_gate_big(const Args& a, uint32_t gate, uint4 in, uint32_t v, uint32_t qdst) {
    const uint4 hi = __ldg(a.dhi + gate);
    const uint32_t r[8] = {in.x, in.y, in.z, in.w, hi.x, hi.y, hi.z, hi.w};
    const uint4 t01 = __ldg(a.dtt + 2 * (uint64_t)gate), t23 = __ldg(a.dtt + 2 * (uint64_t)gate + 1);
    const uint64_t t4[4] = {((uint64_t)t01.y << 32) | t01.x, ((uint64_t)t01.w << 32) | t01.z,
                            ((uint64_t)t23.y << 32) | t23.x, ((uint64_t)t23.w << 32) | t23.z};
    constexpr int NW = sizeof(VT) / 4;
    uint32_t xw[K][NW];
#pragma unroll
    for (int i = 0; i < K; ++i) {
        const VT xv = __ldg(reinterpret_cast<const VT*>(a.state + (uint64_t)resolve(r[i], a.qcur) * a.stride) + v);
        const uint32_t* xp = reinterpret_cast<const uint32_t*>(&xv);
#pragma unroll
        for (int j = 0; j < NW; ++j) xw[i][j] = xp[j];
    }
    VT y;
    uint32_t* yp = reinterpret_cast<uint32_t*>(&y);
#pragma unroll
    for (int j = 0; j < NW; ++j) {
        uint32_t xs[K];
#pragma unroll
        for (int i = 0; i < K; ++i) xs[i] = xw[i][j];
        yp[j] = lut_eval_big<K>(t4, xs);
    }
    *(reinterpret_cast<VT*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + v) = y;
    if (qdst != 0xFFFFFFFFu) *(reinterpret_cast<VT*>(a.state + (uint64_t)(qdst + a.qnext) * a.stride) + v) = y;
}

template <int K>
__device__ __forceinline__ void lut_gate_vec16(const LevelArgs& a, uint32_t gate, uint4 in, uint32_t v,
                                               uint64_t tt, uint32_t qdst) {
    uint32_t r[6];
    r[0] = in.x; r[1] = in.y; r[2] = in.z; r[3] = in.w;
    if (K > 4) {
        const uint4 hi = __ldg(a.dhi + gate);
        r[4] = hi.x; r[5] = hi.y;
    }
    uint4 x[K];
#pragma unroll
    for (int i = 0; i < K; ++i) {
        const uint32_t row = resolve(r[i], a.qcur);
        x[i] = __ldg(reinterpret_cast<const uint4*>(a.state + (uint64_t)row * a.stride) + v);
    }
    const uint4 y = lut_eval4<K>(tt, x);
    *(reinterpret_cast<uint4*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + v) = y;
    if (qdst != 0xFFFFFFFFu)
        *(reinterpret_cast<uint4*>(a.state + (uint64_t)(qdst + a.qnext) * a.stride) + v) = y;
}

template <int K>
__device__ __forceinline__ void lut_gate_vec8(const LevelArgs& a, uint32_t gate, uint4 in, uint32_t v,
                                              uint64_t tt, uint32_t qdst) {
    uint32_t r[6];
    r[0] = in.x; r[1] = in.y; r[2] = in.z; r[3] = in.w;
    if (K > 4) {
        const uint4 hi = __ldg(a.dhi + gate);
        r[4] = hi.x; r[5] = hi.y;
    }
    uint2 x[K];
#pragma unroll
    for (int i = 0; i < K; ++i) {
        const uint32_t row = resolve(r[i], a.qcur);
        x[i] = __ldg(reinterpret_cast<const uint2*>(a.state + (uint64_t)row * a.stride) + v);
    }
    uint32_t xs[K];
    uint2 y;
#pragma unroll
    for (int i = 0; i < K; ++i) xs[i] = x[i].x;
    y.x = lut_eval<K>(tt, xs);
#pragma unroll
    for (int i = 0; i < K; ++i) xs[i] = x[i].y;
    y.y = lut_eval<K>(tt, xs);
    *(reinterpret_cast<uint2*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + v) = y;
    if (qdst != 0xFFFFFFFFu)
        *(reinterpret_cast<uint2*>(a.state + (uint64_t)(qdst + a.qnext) * a.stride) + v) = y;
}

// One thread = one gate x one vector (16 B = 128 stimuli, or 8 B = 64 when a row has an
// odd number of words).  vpr = vectors per row; when vpr >= 32 every warp works on a
// single gate (k is warp-uniform, loads are 512 B contiguous per input row).
template <bool VEC16, bool POW2>
__global__ void __launch_bounds__(256) k_level_lut(LevelArgs a, uint32_t vpr, uint32_t vshift) {
    pdl_entry();
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t gi = POW2 ? (t >> vshift) : (t / vpr);
    if (gi >= a.ng) return;
    const uint32_t v = POW2 ? (t & (vpr - 1)) : (t - gi * vpr);
    const uint32_t gate = a.g0 + gi;
    const uint4 in = __ldg(a.din + gate);
    const uint4 au = __ldg(reinterpret_cast<const uint4*>(a.aux) + gate);
    const uint64_t tt = ((uint64_t)au.y << 32) | au.x;
    const uint32_t qdst = au.z, k = au.w & 0xFFu;
    if (VEC16) {
        switch (k) {
            case 1: lut_gate_vec16<1>(a, gate, in, v, tt, qdst); break;
            case 2: lut_gate_vec16<2>(a, gate, in, v, tt, qdst); break;
            case 3: lut_gate_vec16<3>(a, gate, in, v, tt, qdst); break;
            case 4: lut_gate_vec16<4>(a, gate, in, v, tt, qdst); break;
            case 5: lut_gate_vec16<5>(a, gate, in, v, tt, qdst); break;
            case 6: lut_gate_vec16<6>(a, gate, in, v, tt, qdst); break;
            case 7: lut_gate_big<7, uint4>(a, gate, in, v, qdst); break;
            default: lut_gate_big<8, uint4>(a, gate, in, v, qdst); break;
        }
    } else {
        switch (k) {
            case 1: lut_gate_vec8<1>(a, gate, in, v, tt, qdst); break;
            case 2: lut_gate_vec8<2>(a, gate, in, v, tt, qdst); break;
            case 3: lut_gate_vec8<3>(a, gate, in, v, tt, qdst); break;
            case 4: lut_gate_vec8<4>(a, gate, in, v, tt, qdst); break;
            case 5: lut_gate_vec8<5>(a, gate, in, v, tt, qdst); break;
            case 6: lut_gate_vec8<6>(a, gate, in, v, tt, qdst); break;
            case 7: lut_gate_big<7, uint2>(a, gate, in, v, qdst); break;
            default: lut_gate_big<8, uint2>(a, gate, in, v, qdst); break;
        }
    }
}

// Wide-row variant: every warp owns one gate and U x 32 consecutive 16-byte vectors of
// it; all U*k input loads are issued before any is consumed (memory-level parallelism
// U*k per thread, one descriptor fetch per U vectors).  HINT: L2 eviction priority per
// store (aux.k bit 8 = "a gate of the next level reads this row": evict_last; other rows
// and the register next-bank store: evict_first).
template <int K, int U, bool HINT>
__device__ __forceinline__ void lut_gate_u(const LevelArgs& a, uint32_t gate, uint4 in, uint32_t v0,
                                           uint64_t tt, uint32_t qdst, bool hot) {
    uint32_t r[6];
    r[0] = in.x; r[1] = in.y; r[2] = in.z; r[3] = in.w;
    if (K > 4) {
        const uint4 hi = __ldg(a.dhi + gate);
        r[4] = hi.x; r[5] = hi.y;
    }
    const uint4* src[K];
#pragma unroll
    for (int i = 0; i < K; ++i)
        src[i] = reinterpret_cast<const uint4*>(a.state + (uint64_t)resolve(r[i], a.qcur) * a.stride) + v0;
    uint4 x[U][K];
    uint64_t pf = 0;
    if (HINT) pf = l2_policy_first();
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
        for (int i = 0; i < K; ++i) x[u][i] = (HINT && a.hint_ld) ? ld_hint(src[i] + u * 32, pf) : __ldg(src[i] + u * 32);
    uint4* dst = reinterpret_cast<uint4*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + v0;
    // fused latch target: a boolean, never a null pointer plus an offset (the compiler may
    // assume such a pointer non-null and drop the test; seen with the L2-hint stores)
    const bool latch = qdst != 0xFFFFFFFFu;
    uint4* qd = reinterpret_cast<uint4*>(a.state + (uint64_t)((latch ? qdst : 0u) + a.qnext) * a.stride) + v0;
    uint64_t po = 0;
    if (HINT) po = hot ? l2_policy_last() : pf;
#pragma unroll
    for (int u = 0; u < U; ++u) {
        const uint4 y = lut_eval4<K>(tt, x[u]);
        if (HINT) {
            st_hint(dst + u * 32, y, po);
            st_hint_if(qd + u * 32, y, pf, latch);
        } else {
            dst[u * 32] = y;
            if (latch) qd[u * 32] = y;
        }
    }
}

// Grid-stride over warp units (gate, chunk of U*32 vectors): the grid is sized to the
// resident capacity (148 SMs x CTAs per SM, a.grid_blocks), so no level ends with a
// partially filled wave of CTAs.
#ifndef GS_U1_MINB
#define GS_U1_MINB 4
#endif
template <int U, bool HINT>
__global__ void __launch_bounds__(256, U > 4 ? 2 : U == 1 ? GS_U1_MINB : 4)
    k_level_lut_wide(LevelArgs a, uint32_t cpg_shift, uint32_t vec0) {
    pdl_entry();
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t total = a.ng << cpg_shift;
    const uint32_t stride = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; warp < total; warp += stride) {
        const uint32_t gi = warp >> cpg_shift;
        const uint32_t chunk = warp & ((1u << cpg_shift) - 1);
        const uint32_t v0 = vec0 + chunk * 32 * U + lane;
        const uint32_t gate = a.g0 + gi;
        const uint4 in = __ldg(a.din + gate);
        const uint4 au = __ldg(reinterpret_cast<const uint4*>(a.aux) + gate);
        const uint64_t tt = ((uint64_t)au.y << 32) | au.x;
        const uint32_t qdst = au.z, k = au.w & 0xFFu;
        const bool hot = (au.w >> 8) & 1u;
        switch (k) {
            case 1: lut_gate_u<1, U, HINT>(a, gate, in, v0, tt, qdst, hot); break;
            case 2: lut_gate_u<2, U, HINT>(a, gate, in, v0, tt, qdst, hot); break;
            case 3: lut_gate_u<3, U, HINT>(a, gate, in, v0, tt, qdst, hot); break;
            case 4: lut_gate_u<4, U, HINT>(a, gate, in, v0, tt, qdst, hot); break;
            case 5: lut_gate_u<5, 1, HINT>(a, gate, in, v0, tt, qdst, hot);
                    if (U > 1) lut_gate_u<5, 1, HINT>(a, gate, in, v0 + 32, tt, qdst, hot);
                    if (U > 2) { lut_gate_u<5, 1, HINT>(a, gate, in, v0 + 64, tt, qdst, hot);
                                 lut_gate_u<5, 1, HINT>(a, gate, in, v0 + 96, tt, qdst, hot); }
                    if (U > 4)
                        for (int u = 4; u < U; ++u) lut_gate_u<5, 1, HINT>(a, gate, in, v0 + 32 * u, tt, qdst, hot);
                    break;
            case 6: lut_gate_u<6, 1, HINT>(a, gate, in, v0, tt, qdst, hot);
                    if (U > 1) lut_gate_u<6, 1, HINT>(a, gate, in, v0 + 32, tt, qdst, hot);
                    if (U > 2) { lut_gate_u<6, 1, HINT>(a, gate, in, v0 + 64, tt, qdst, hot);
                                 lut_gate_u<6, 1, HINT>(a, gate, in, v0 + 96, tt, qdst, hot); }
                    if (U > 4)
                        for (int u = 4; u < U; ++u) lut_gate_u<6, 1, HINT>(a, gate, in, v0 + 32 * u, tt, qdst, hot);
                    break;
            case 7:
#pragma unroll 1
                    for (int u = 0; u < U; ++u) lut_gate_big<7, uint4>(a, gate, in, v0 + 32 * u, qdst);
                    break;
            default:
#pragma unroll 1
                    for (int u = 0; u < U; ++u) lut_gate_big<8, uint4>(a, gate, in, v0 + 32 * u, qdst);
                    break;
        }
    }
}

// ------------------------------------------- kernel A, bulk-copy (TMA) staged gathers
// The same evaluation as k_level_lut_wide, but a gate's input rows reach the SM through
// the bulk-copy engine instead of per-thread loads: a work item is (gate, C-byte chunk of
// its rows); one producer warp per CTA streams the level's descriptors (32 items per
// coalesced batch, the next batch prefetched), waits for a free stage of an S-deep ring in
// shared memory, arms the stage's mbarrier with k*C transaction bytes and issues k
// cp.async.bulk copies of C contiguous bytes; eight consumer warps wait on the stage's
// mbarrier, evaluate the truth table on the staged bits (LDS.128, bank-conflict free),
// store the output row (and the fused latch row) with coalesced 16-byte stores and release
// the stage.  Whole-row-sized copies keep each input row's DRAM pages together; measured
// on the access pattern alone (scripts/micro/gather_bulk.cu) this reaches 6.45 TB/s for
// three random 8 KB input rows + one output row, against 4.5-5.3 TB/s for the register
// gather.  Only levels whose gates all have 1 <= k <= 4 take this path.
constexpr uint32_t BULK_THREADS = 288;          // 8 consumer warps + 1 producer warp

__device__ __forceinline__ void mbar_init_d(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(bar)),
                 "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_wait_d(uint64_t* bar, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"((uint32_t)__cvta_generic_to_shared(bar)), "r"(parity), "r"(1000000u)   // suspend, not spin
            : "memory");
    }
}

template <int K, int C>
__device__ __forceinline__ void bulk_eval(const uint4* stage, uint8_t* dst, uint8_t* qd, bool latch, uint64_t tt,
                                          uint32_t t) {
#pragma unroll
    for (uint32_t v = t; v < C / 16; v += 256) {
        uint4 x[K];
#pragma unroll
        for (int i = 0; i < K; ++i) x[i] = stage[i * (C / 16) + v];
        const uint4 y = lut_eval4<K>(tt, x);
        reinterpret_cast<uint4*>(dst)[v] = y;
        if (latch) reinterpret_cast<uint4*>(qd)[v] = y;
    }
}

template <int C, int S, int MINB>
__global__ void __launch_bounds__(BULK_THREADS, MINB) k_level_bulk(LevelArgs a, uint32_t cpg_shift, uint32_t byte0) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem);          // [S] data landed
    uint64_t* empty = full + S;                                  // [S] consumers done
    uint4* hdr = reinterpret_cast<uint4*>(smem + 16 * S);        // [S] {tt lo, tt hi, qdst, k}
    uint4* buf = reinterpret_cast<uint4*>(smem + 1024);          // [S][4][C]
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init_d(&full[s], 1);
            mbar_init_d(&empty[s], 8);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    pdl_entry();
    const uint32_t total = a.ng << cpg_shift, cmask = (1u << cpg_shift) - 1u, G = gridDim.x;
    if (warp == 8) {                                             // ---- producer warp
        uint32_t j = 0;
        uint32_t it = blockIdx.x + lane * G;
        uint4 in = make_uint4(0, 0, 0, 0), au = make_uint4(0, 0, 0, 0);
        if (it < total) {
            in = __ldg(a.din + a.g0 + (it >> cpg_shift));
            au = __ldg(reinterpret_cast<const uint4*>(a.aux) + a.g0 + (it >> cpg_shift));
        }
        for (uint32_t base = blockIdx.x; base < total; base += 32 * G) {
            const uint32_t nit = base + 32 * G + lane * G;       // prefetch the next batch
            uint4 in_n = make_uint4(0, 0, 0, 0), au_n = make_uint4(0, 0, 0, 0);
            if (nit < total) {
                in_n = __ldg(a.din + a.g0 + (nit >> cpg_shift));
                au_n = __ldg(reinterpret_cast<const uint4*>(a.aux) + a.g0 + (nit >> cpg_shift));
            }
            const uint32_t n = min(32u, (total - base + G - 1) / G);
            for (uint32_t i = 0; i < n; ++i, ++j) {
                const uint32_t r0 = __shfl_sync(FULL, in.x, i), r1 = __shfl_sync(FULL, in.y, i);
                const uint32_t r2 = __shfl_sync(FULL, in.z, i), r3 = __shfl_sync(FULL, in.w, i);
                const uint32_t t0 = __shfl_sync(FULL, au.x, i), t1 = __shfl_sync(FULL, au.y, i);
                const uint32_t qd = __shfl_sync(FULL, au.z, i), kw = __shfl_sync(FULL, au.w, i);
                if (lane == 0) {
                    const uint32_t s = j % S;
                    if (j >= S) mbar_wait_d(&empty[s], ((j / S) - 1) & 1);
                    const uint32_t k = kw & 0xFFu;
                    hdr[s] = make_uint4(t0, t1, qd, k);
                    const uint64_t off = byte0 + (uint64_t)((base + i * G) & cmask) * C;
                    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&full[s]);
                    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(k * C)
                                 : "memory");
                    const uint32_t rr[4] = {r0, r1, r2, r3};
#pragma unroll
                    for (uint32_t q = 0; q < 4; ++q) {
                        if (q >= k) break;
                        const uint8_t* src = a.state + (uint64_t)resolve(rr[q], a.qcur) * a.stride + off;
                        const uint32_t dst = (uint32_t)__cvta_generic_to_shared(buf + (s * 4 + q) * (C / 16));
                        asm volatile(
                            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                            ::"r"(dst), "l"(src), "r"((uint32_t)C), "r"(bar)
                            : "memory");
                    }
                }
                __syncwarp();
            }
            in = in_n;
            au = au_n;
        }
        return;
    }
    // ---- consumer warps 0..7
    const uint32_t t = threadIdx.x;
    uint32_t j = 0;
    for (uint32_t it = blockIdx.x; it < total; it += G, ++j) {
        const uint32_t s = j % S;
        mbar_wait_d(&full[s], (j / S) & 1);
        const uint4 h = hdr[s];
        const uint64_t tt = ((uint64_t)h.y << 32) | h.x;
        const uint32_t gate = a.g0 + (it >> cpg_shift);
        const uint64_t off = byte0 + (uint64_t)(it & cmask) * C;
        uint8_t* dst = a.state + (uint64_t)(a.row_gate0 + gate) * a.stride + off;
        const bool latch = h.z != 0xFFFFFFFFu;             // (never a null pointer + offset)
        uint8_t* qd = a.state + (uint64_t)((latch ? h.z : 0u) + a.qnext) * a.stride + off;
        const uint4* st = buf + s * 4 * (C / 16);
        switch (h.w) {
            case 1: bulk_eval<1, C>(st, dst, qd, latch, tt, t); break;
            case 2: bulk_eval<2, C>(st, dst, qd, latch, tt, t); break;
            case 3: bulk_eval<3, C>(st, dst, qd, latch, tt, t); break;
            default: bulk_eval<4, C>(st, dst, qd, latch, tt, t); break;
        }
        __syncwarp();
        if (lane == 0)
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&empty[s]))
                         : "memory");
    }
}

template <int C, int S, int MINB>
static cudaError_t launch_bulk(const LevelArgs& a, cudaStream_t st, int sms) {
    constexpr size_t smem = 1024 + (size_t)S * 4 * C;
    static std::atomic<uint64_t> attr{0};     // devices whose function attribute is set
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const uint64_t bit = 1ull << (dev & 63);
    if (!(attr.load() & bit)) {
        e = cudaFuncSetAttribute(k_level_bulk<C, S, MINB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr.fetch_or(bit);
    }
    const uint32_t vrow = a.vslab ? a.vslab : a.words / 2;
    const uint32_t cpg = vrow * 16 / C;
    uint32_t sh = 0;
    while ((1u << sh) < cpg) ++sh;
    const uint64_t items = (uint64_t)a.ng << sh;
    if (items >= (1ull << 31)) return cudaErrorInvalidValue;
    const uint32_t grid = (uint32_t)std::min<uint64_t>(items, (uint64_t)sms * MINB);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(BULK_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = a.pdl ? at : nullptr;
    cfg.numAttrs = a.pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, k_level_bulk<C, S, MINB>, a, sh, a.vec0 * 16u);
}

uint32_t level_bulk_chunk(uint32_t words, uint32_t vslab) {
    if (words % 2) return 0;
    const uint64_t bytes = vslab ? (uint64_t)vslab * 16 : (uint64_t)words * 8;
    for (uint32_t c : {8192u, 4096u, 2048u}) {
        if (bytes % c) continue;
        const uint64_t cpg = bytes / c;
        if ((cpg & (cpg - 1)) == 0) return c;
    }
    return 0;
}

cudaError_t launch_level_bulk(const LevelArgs& a, cudaStream_t s) {
    if (a.ng == 0) return cudaSuccess;
    const int sms = a.sms ? (int)a.sms : 148;
    switch (level_bulk_chunk(a.words, a.vslab)) {     // (chunk, stages, CTAs/SM): measured best
        case 8192: return launch_bulk<8192, 3, 2>(a, s, sms);
        case 4096: return launch_bulk<4096, 4, 3>(a, s, sms);
        case 2048: return launch_bulk<2048, 6, 3>(a, s, sms);
        default: return cudaErrorInvalidValue;
    }
}

uint32_t level_lut_resident_blocks(int device) {
    int sms = 0, per = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) return 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_level_lut_wide<4, false>, 256, 0) != cudaSuccess)
        return 0;
    return (uint32_t)(sms * per);
}

cudaError_t launch_level_lut(const LevelArgs& a, cudaStream_t s) {
    if (a.ng == 0) return cudaSuccess;
    if (a.bulk && level_bulk_chunk(a.words, a.vslab)) return launch_level_bulk(a, s);
    // slab: 16-byte vectors [a.vec0, a.vec0 + a.vslab) of every row (whole row if vslab == 0)
    if ((a.words % 2) == 0) {
        const uint32_t vrow = a.vslab ? a.vslab : a.words / 2;
        for (uint32_t U : {8u, 4u, 2u, 1u}) {
            if (U == 8 && a.unroll != 8) continue;              // U = 8 only on request
            if (a.unroll && U > a.unroll) continue;
            const uint32_t cpg = vrow / (32 * U);
            if (vrow % (32 * U) || cpg == 0 || (cpg & (cpg - 1))) continue;
            // auto: trade vectors per thread for warps while a narrow level would not
            // fill the GPU (memory-level parallelism per thread vs threads in flight)
            if (!a.unroll && U > 1 && (uint64_t)a.ng * cpg < a.min_warps) continue;
            uint32_t sh = 0;
            while ((1u << sh) < cpg) ++sh;
            const uint64_t threads = ((uint64_t)a.ng << sh) * 32;
            if (threads >= (1ull << 31)) break;
            uint32_t blocks = (uint32_t)((threads + 255) / 256);
            // grid-stride at the resident capacity when the level is only a few waves deep (a
            // partial last wave would idle SMs for a large share of the launch; measured: C3
            // +8.5 %); deep levels (C4: 12 waves, C5: 41) keep one CTA per chunk (-1 % otherwise)
            const uint32_t cap = U == 1 ? a.grid_blocks / 4 * GS_U1_MINB : a.grid_blocks;   // resident CTAs
            if (cap && blocks > cap && blocks <= 4 * cap) blocks = cap;
            if (U == 8) return launch_k(k_level_lut_wide<8, false>, blocks, s, a.pdl, a, sh, a.vec0);
            if (a.hint) {
                if (U == 4) return launch_k(k_level_lut_wide<4, true>, blocks, s, a.pdl, a, sh, a.vec0);
                if (U == 2) return launch_k(k_level_lut_wide<2, true>, blocks, s, a.pdl, a, sh, a.vec0);
                return launch_k(k_level_lut_wide<1, true>, blocks, s, a.pdl, a, sh, a.vec0);
            }
            if (U == 4) return launch_k(k_level_lut_wide<4, false>, blocks, s, a.pdl, a, sh, a.vec0);
            if (U == 2) return launch_k(k_level_lut_wide<2, false>, blocks, s, a.pdl, a, sh, a.vec0);
            return launch_k(k_level_lut_wide<1, false>, blocks, s, a.pdl, a, sh, a.vec0);
        }
    }
    if (a.vslab) return cudaErrorInvalidValue;      // slabs only on the wide path
    const bool vec16 = (a.words % 2) == 0;
    const uint32_t vpr = vec16 ? a.words / 2 : a.words;
    const bool pow2 = (vpr & (vpr - 1)) == 0;
    uint32_t vshift = 0;
    while ((1u << vshift) < vpr) ++vshift;
    const uint64_t threads = (uint64_t)a.ng * vpr;
    if (threads >= (1ull << 31)) return cudaErrorInvalidValue;
    const uint32_t blocks = (uint32_t)((threads + 255) / 256);
    if (vec16) {
        if (pow2) return launch_k(k_level_lut<true, true>, blocks, s, a.pdl, a, vpr, vshift);
        return launch_k(k_level_lut<true, false>, blocks, s, a.pdl, a, vpr, vshift);
    }
    if (pow2) return launch_k(k_level_lut<false, true>, blocks, s, a.pdl, a, vpr, vshift);
    return launch_k(k_level_lut<false, false>, blocks, s, a.pdl, a, vpr, vshift);
}

// ------------------------------------------- kernel A, persistent slab dataflow ("D")
// One launch evaluates every level of one cycle.  The lanes are cut into slabs of
// 4096*VPL stimuli (512*VPL bytes per row); slabs are independent, so the levels of
// different slabs need no ordering.  Work items (slab, level, chunk of 8*gpw gates)
// are handed out in a fixed order through one atomic queue head; an item waits only
// until every item of the previous level of ITS slab is done (a per-(slab, level)
// counter, release/acquire).  Consequences:
//   * no launch boundary per level: the tail of level l of slab s overlaps level l
//     of slab s+1 (slabs are walked `interleave` at a time, level-major);
//   * a slab's recent levels (~15k gates x 512 B per level on C4) stay in L2, so most
//     gate-input reads (inputs from level l-1..l-8) are L2 hits rather than HBM reads;
//   * no deadlock for any grid size: an item only waits for items taken earlier from
//     the queue, which are held by running CTAs (induction on the queue index).
// Loads use ld.global.cg (L2, never a stale L1 line); stores are plain.
__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// A gate's slab row segment (slab_vec 16-byte vectors) is owned by a group of LPG
// lanes, each holding VPT = slab_vec / LPG vectors, so every thread keeps VPT * k
// independent loads in flight (the memory-level parallelism of kernel A's U = 4) and
// a warp works on 32 / LPG gates at once.
template <int K, int VPT, int LPG>
__device__ __forceinline__ void df_gate(const DfArgs& a, uint32_t gate, uint4 in, uint64_t tt, uint32_t qdst,
                                        uint32_t v0) {
    uint32_t r[6];
    r[0] = in.x; r[1] = in.y; r[2] = in.z; r[3] = in.w;
    if (K > 4) {
        const uint4 hi = __ldg(a.dhi + gate);
        r[4] = hi.x; r[5] = hi.y;
    }
    const uint4* src[K];
#pragma unroll
    for (int i = 0; i < K; ++i)
        src[i] = reinterpret_cast<const uint4*>(a.state + (uint64_t)resolve(r[i], a.qcur) * a.stride) + v0;
    uint4 x[VPT][K];
#pragma unroll
    for (int u = 0; u < VPT; ++u)
#pragma unroll
        for (int i = 0; i < K; ++i) x[u][i] = __ldcg(src[i] + u * LPG);
    uint4* dst = reinterpret_cast<uint4*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + v0;
    // fused latch target: a boolean, never a null pointer plus an offset (the compiler may
    // assume such a pointer non-null and drop the test; seen with the L2-hint stores)
    const bool latch = qdst != 0xFFFFFFFFu;
    uint4* qd = reinterpret_cast<uint4*>(a.state + (uint64_t)((latch ? qdst : 0u) + a.qnext) * a.stride) + v0;
#pragma unroll
    for (int u = 0; u < VPT; ++u) {
        const uint4 y = lut_eval4<K>(tt, x[u]);
        dst[u * LPG] = y;
        if (latch) qd[u * LPG] = y;
    }
}

// k = 5, 6: one vector at a time (keeps the register footprint of k <= 4)
template <int K, int VPT, int LPG>
__device__ __forceinline__ void df_gate_wide(const DfArgs& a, uint32_t gate, uint4 in, uint64_t tt, uint32_t qdst,
                                             uint32_t v0) {
#pragma unroll 1
    for (int u = 0; u < VPT; ++u) df_gate<K, 1, LPG>(a, gate, in, tt, qdst, v0 + u * LPG);
}

// Work item = (slab, level, chunk of 8 * gpw gates) for one CTA (8 warps x gpw gates).
// Items are numbered groups of `interleave` slabs -> level -> slab -> chunk and handed
// out by one atomic queue head; the claim of the next item is issued while the current
// one is processed.  No deadlock for any grid size: an item only waits for items
// claimed earlier, which are held by running CTAs (induction on the queue index).
template <int VPT, int LPG>
__global__ void __launch_bounds__(256, 4) k_dataflow(DfArgs a) {
    pdl_entry();
    __shared__ unsigned s_item[2];
    constexpr uint32_t GPP = 32 / LPG;                            // gates per warp pass
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t grp = lane / LPG, li = lane % LPG;
    const uint32_t per_group = a.interleave * a.items_per_slab;
    if (threadIdx.x == 0) s_item[0] = atomicAdd(a.qhead, 1u);
    __syncthreads();
    for (uint32_t it = 0;; it ^= 1) {
        const uint32_t q = s_item[it];
        if (q >= a.total_items) return;                           // block-uniform
        unsigned next = 0;
        if (threadIdx.x == 0) next = atomicAdd(a.qhead, 1u);      // in flight during the item
        // ---- decode q -> (slab, level, chunk)
        const uint32_t sg = q / per_group;
        uint32_t rr = q - sg * per_group;
        const uint32_t s0 = sg * a.interleave;
        const uint32_t I = min(a.interleave, a.n_slabs - s0);
        uint32_t lo = 0, hi = a.nl;                               // I*item0[lo] <= rr < I*item0[hi]
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (I * __ldg(a.lv_item0 + mid) <= rr) lo = mid; else hi = mid;
        }
        const uint32_t l = lo;
        const uint32_t it0 = __ldg(a.lv_item0 + l);
        const uint32_t nli = __ldg(a.lv_item0 + l + 1) - it0;
        rr -= I * it0;
        const uint32_t si = rr / nli, chunk = rr - si * nli;
        const uint32_t slab = s0 + si;
        // ---- this warp's gates and their descriptors (issued before the wait)
        const uint32_t lg1 = __ldg(a.lv_gate0 + l + 1);
        const uint32_t gb = __ldg(a.lv_gate0 + l) + (chunk * 8 + warp) * a.gpw;
        const uint32_t ge = min(gb + a.gpw, lg1);
        uint4 my_in = make_uint4(0, 0, 0, 0), my_au = make_uint4(0, 0, 0, 0);
        if (gb + lane < ge) {
            my_in = __ldg(a.din + gb + lane);
            my_au = __ldg(reinterpret_cast<const uint4*>(a.aux) + gb + lane);
        }
        // ---- wait until every item of the previous level of this slab is done
        if (l > 0) {
            if (threadIdx.x == 0) {
                const unsigned need = it0 - __ldg(a.lv_item0 + l - 1);
                const unsigned* p = a.done + (uint64_t)slab * a.nl + (l - 1);
                if (ld_acquire(p) < need) {
                    const long long t0 = clock64();
                    while (ld_acquire(p) < need) {
                        __nanosleep(64);
                        if (clock64() - t0 > (1ll << 35)) __trap();   // ~17 s: never hang the GPU
                    }
                }
            }
            __syncthreads();
        }
        const uint32_t v0 = slab * a.slab_vec + li;
        for (uint32_t p0 = 0; gb + p0 < ge; p0 += GPP) {
            const uint32_t j = p0 + grp;
            uint4 in, au;
            in.x = __shfl_sync(FULL, my_in.x, j & 31); in.y = __shfl_sync(FULL, my_in.y, j & 31);
            in.z = __shfl_sync(FULL, my_in.z, j & 31); in.w = __shfl_sync(FULL, my_in.w, j & 31);
            au.x = __shfl_sync(FULL, my_au.x, j & 31); au.y = __shfl_sync(FULL, my_au.y, j & 31);
            au.z = __shfl_sync(FULL, my_au.z, j & 31); au.w = __shfl_sync(FULL, my_au.w, j & 31);
            if (gb + j >= ge) continue;
            const uint32_t g = gb + j;
            const uint64_t tt = ((uint64_t)au.y << 32) | au.x;
            switch (au.w & 0xFFu) {
                case 1: df_gate<1, VPT, LPG>(a, g, in, tt, au.z, v0); break;
                case 2: df_gate<2, VPT, LPG>(a, g, in, tt, au.z, v0); break;
                case 3: df_gate<3, VPT, LPG>(a, g, in, tt, au.z, v0); break;
                case 4: df_gate<4, VPT, LPG>(a, g, in, tt, au.z, v0); break;
                case 5: df_gate_wide<5, VPT, LPG>(a, g, in, tt, au.z, v0); break;
                case 6: df_gate_wide<6, VPT, LPG>(a, g, in, tt, au.z, v0); break;
                case 7:
#pragma unroll 1
                    for (int u = 0; u < VPT; ++u) lut_gate_big<7, uint4>(a, g, in, v0 + u * LPG, au.z);
                    break;
                default:
#pragma unroll 1
                    for (int u = 0; u < VPT; ++u) lut_gate_big<8, uint4>(a, g, in, v0 + u * LPG, au.z);
                    break;
            }
        }
        if (threadIdx.x == 0) s_item[it ^ 1] = next;
        // ---- publish: all of this item's stores happen-before the counter increment
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(a.done + (uint64_t)slab * a.nl + l, 1u);
        }
    }
}

// slab_vec = 16-byte vectors per slab row (32, 64 or 128); lanes per gate = slab_vec / 4
#define DF_SWITCH(SV, CALL)                                                  \
    switch (SV) {                                                            \
        case 32: CALL(4, 8); break;                                          \
        case 64: CALL(4, 16); break;                                         \
        case 128: CALL(4, 32); break;                                        \
        default: return cudaErrorInvalidValue;                               \
    }

cudaError_t dataflow_grid(uint32_t slab_vec, int device, uint32_t* grid) {
    int sms = 0, per = 0;
    cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    if (e != cudaSuccess) return e;
#define DF_OCC(V, L) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_dataflow<V, L>, 256, 0)
    DF_SWITCH(slab_vec, DF_OCC)
#undef DF_OCC
    if (e != cudaSuccess) return e;
    *grid = (uint32_t)(sms * (per > 0 ? per : 1));
    return cudaSuccess;
}

cudaError_t launch_dataflow(const DfArgs& a, uint32_t grid, cudaStream_t s) {
    if (a.total_items == 0) return cudaSuccess;
    cudaError_t e = cudaSuccess;
#define DF_LAUNCH(V, L) e = launch_k(k_dataflow<V, L>, grid, s, 0u, a)
    DF_SWITCH(a.slab_vec, DF_LAUNCH)
#undef DF_LAUNCH
    return e;
}

// ------------------------------------------------------------ kernel B: polynomial
// The paper's two-layer network per gate (Fig. 2; Eq. 1-3) in exact integer
// arithmetic, BIT-SLICED: one thread holds 32 stimuli (one 32-bit word of every input row)
// and evaluates, for every nonzero monomial S (the sparse polynomial):
//   hidden neuron  h_S = Theta(sum_{s in S} x_s - |S| + 1): the sum is a 4-plane bit-sliced
//                  counter of the selected inputs, compared with |S| - 1 (it cannot exceed
//                  |S|, so "> |S| - 1" is "== |S|");
//   output neuron  acc += w_S h_S: a two's-complement accumulator of B bit-planes
//                  (|acc| <= sum |w_S| <= 3^k: B = 8 for k <= 4, 16 for k <= 8), the
//                  constant w_S added under the mask h_S one set bit of |w_S| at a time
//                  (half-adder / half-subtractor ripples that stop once no lane carries).
// The gate's output is [acc == 1]; lanes with acc outside {0, 1} are counted (P:224 says
// there are none).  check_only: compare with the row kernel A wrote (GS_KERNEL_AB).
template <int B, int KMAX>
__device__ __forceinline__ void poly_word(const LevelArgs& a, uint32_t gate, uint32_t j, uint32_t k, uint32_t qdst,
                                          const uint32_t* r, int check_only, uint32_t& bad) {
    // j = 64-bit word: the thread holds 64 stimuli as two 32-lane words (NW = 2), so the
    // term decode and its branches are shared by both
    constexpr int NW = 2;
    uint32_t x[KMAX][NW];
#pragma unroll
    for (int i = 0; i < KMAX; ++i) {
        uint2 v = make_uint2(0u, 0u);
        if (i < (int)k)
            v = __ldg(reinterpret_cast<const uint2*>(a.state + (uint64_t)resolve(r[i], a.qcur) * a.stride) + j);
        x[i][0] = v.x;
        x[i][1] = v.y;
    }
    uint32_t acc[B][NW];
#pragma unroll
    for (int b = 0; b < B; ++b) acc[b][0] = acc[b][1] = 0u;
    const uint32_t t0 = __ldg(a.term_off + gate), t1 = __ldg(a.term_off + gate + 1);
    for (uint32_t ti = t0; ti < t1; ++ti) {
        const uint32_t tm = __ldg(a.terms + ti);
        const uint32_t S = tm & 0xFFu;                          // monomial S (bit s <-> x_s)
        const uint32_t nS = (uint32_t)((int)(int8_t)((tm >> 8) & 0xFFu) + 1);   // |S| (bias + 1, Eq. 3)
        const int w = (int)(int16_t)(tm >> 16);                 // w_S (Eq. 1)
        // hidden neuron: bit-sliced sum of the selected inputs (4-plane counter; a carry
        // ripple stops as soon as no lane carries), then the threshold "sum > |S| - 1"
        uint32_t c[4][NW] = {{0u, 0u}, {0u, 0u}, {0u, 0u}, {0u, 0u}};
#pragma unroll
        for (int i = 0; i < KMAX; ++i) {
            if ((S >> i) & 1u) {
                uint32_t cy0 = x[i][0], cy1 = x[i][1];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const uint32_t u0 = c[q][0] & cy0, u1 = c[q][1] & cy1;
                    c[q][0] ^= cy0;
                    c[q][1] ^= cy1;
                    cy0 = u0;
                    cy1 = u1;
                    if (!(cy0 | cy1)) break;
                }
            }
        }
        // the sum cannot exceed |S|, so "> |S| - 1" is "== |S|": compare the planes with |S|
        const uint32_t m0 = 0u - (nS & 1u), m1 = 0u - ((nS >> 1) & 1u), m2 = 0u - ((nS >> 2) & 1u),
                       m3 = 0u - ((nS >> 3) & 1u);
        uint32_t h[NW];
#pragma unroll
        for (int n = 0; n < NW; ++n)
            h[n] = ~((c[0][n] ^ m0) | (c[1][n] ^ m1) | (c[2][n] ^ m2) | (c[3][n] ^ m3));
        // output neuron: acc += w_S * h_S in two's complement (mod 2^B): for every set bit p
        // of |w_S|, add (w_S > 0) or subtract (w_S < 0) the mask h at plane p, rippling the
        // carry / borrow upward only while some lane still carries
        const uint32_t aw = (uint32_t)(w < 0 ? -w : w);
        for (uint32_t m = aw; m; m &= m - 1) {
            const int pb = __ffs(m) - 1;
            uint32_t cy0 = h[0], cy1 = h[1];
            if (w > 0) {
#pragma unroll
                for (int b = 0; b < B; ++b) {
                    if (b < pb) continue;
                    const uint32_t u0 = acc[b][0] & cy0, u1 = acc[b][1] & cy1;
                    acc[b][0] ^= cy0;
                    acc[b][1] ^= cy1;
                    cy0 = u0;
                    cy1 = u1;
                    if (!(cy0 | cy1)) break;
                }
            } else {
#pragma unroll
                for (int b = 0; b < B; ++b) {
                    if (b < pb) continue;
                    const uint32_t u0 = ~acc[b][0] & cy0, u1 = ~acc[b][1] & cy1;
                    acc[b][0] ^= cy0;
                    acc[b][1] ^= cy1;
                    cy0 = u0;
                    cy1 = u1;
                    if (!(cy0 | cy1)) break;
                }
            }
        }
    }
    uint32_t one[NW];
#pragma unroll
    for (int n = 0; n < NW; ++n) {
        uint32_t hi = 0u;
#pragma unroll
        for (int b = 1; b < B; ++b) hi |= acc[b][n];
        one[n] = acc[0][n] & ~hi;
        const uint32_t zero = ~(acc[0][n] | hi);
        bad += __popc(~(one[n] | zero));
    }
    const uint2 y = make_uint2(one[0], one[1]);
    uint2* out = reinterpret_cast<uint2*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + j;
    if (check_only) {
        const uint2 ref = *out;
        const uint32_t diff = __popc(ref.x ^ y.x) + __popc(ref.y ^ y.y);
        if (diff) atomicAdd(&a.ctl->ab_mismatch, (unsigned long long)diff);
    } else {
        *out = y;
        if (qdst != 0xFFFFFFFFu) reinterpret_cast<uint2*>(a.state + (uint64_t)(qdst + a.qnext) * a.stride)[j] = y;
    }
}

// one thread = one gate x one 64-bit word (64 stimuli); consecutive threads = consecutive
// words of the same gate (coalesced loads, warp-uniform terms)
__global__ void __launch_bounds__(256) k_level_poly(LevelArgs a, uint32_t words64, int check_only) {
    pdl_entry();
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t gi = (uint32_t)(t / words64), j = (uint32_t)(t - (uint64_t)gi * words64);
    uint32_t bad = 0u;
    if (gi < a.ng) {
        const uint32_t gate = a.g0 + gi;
        const uint4 in = __ldg(a.din + gate);
        const uint4 au = __ldg(reinterpret_cast<const uint4*>(a.aux) + gate);
        const uint32_t qdst = au.z, k = au.w & 0xFFu;          // k <= GS_MAX_K_POLY = 8
        uint32_t r[8] = {in.x, in.y, in.z, in.w, 0u, 0u, 0u, 0u};
        if (k > 4) {
            const uint4 hi = __ldg(a.dhi + gate);
            r[4] = hi.x; r[5] = hi.y; r[6] = hi.z; r[7] = hi.w;
            poly_word<16, 8>(a, gate, j, k, qdst, r, check_only, bad);
        } else {
            poly_word<8, 4>(a, gate, j, k, qdst, r, check_only, bad);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) bad += __shfl_xor_sync(FULL, bad, o);
    if ((threadIdx.x & 31) == 0 && bad) atomicAdd(&a.ctl->violations, (unsigned long long)bad);
}

cudaError_t launch_level_poly(const LevelArgs& a, int check_only, cudaStream_t s) {
    if (a.ng == 0) return cudaSuccess;
    const uint64_t threads = (uint64_t)a.ng * a.words;
    const uint64_t blocks = (threads + 255) / 256;
    if (blocks >= (1ull << 31)) return cudaErrorInvalidValue;
    return launch_k(k_level_poly, (uint32_t)blocks, s, a.pdl, a, a.words, check_only);
}

// --------------------------------------------------------------------- stimulus
__global__ void __launch_bounds__(256) k_stim(Ctl* ctl, uint8_t* state, uint64_t stride, uint32_t words,
                                              uint32_t row_pi0, uint32_t n_pi, uint64_t word_off) {
    pdl_entry();
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (uint64_t)n_pi * words) return;
    const uint32_t p = (uint32_t)(t / words), w = (uint32_t)(t - (uint64_t)p * words);
    const unsigned long long c = ctl->cycle;
    unsigned long long v;
    if (ctl->stim_mode == 0) {
        v = dmix64(dmix64(dmix64(ctl->seed ^ p) ^ c) ^ (word_off + w));
    } else {
        const unsigned long long* src = reinterpret_cast<const unsigned long long*>(ctl->stim_ptr);
        v = src[((c - ctl->stim_base) * n_pi + p) * words + w];
    }
    reinterpret_cast<unsigned long long*>(state + (uint64_t)(row_pi0 + p) * stride)[w] = v;
}

cudaError_t launch_stim(Ctl* ctl, uint8_t* state, uint64_t stride, uint32_t words, uint32_t row_pi0,
                        uint32_t n_pi, uint64_t word_off, uint32_t pdl, cudaStream_t s) {
    const uint64_t n = (uint64_t)n_pi * words;
    if (n == 0) return cudaSuccess;
    return launch_k(k_stim, (uint32_t)((n + 255) / 256), s, pdl, ctl, state, stride, words, row_pi0, n_pi,
                    word_off);
}

// --------------------------------------------------------------- end of cycle
// Blocks [0, latch_blocks): remaining register latches Q_next[r] = src (reads the
// current bank / gate rows, writes the other bank, so order does not matter).
// Blocks [latch_blocks, ...): one warp per word: output MISR (64 bit-planes per word,
// DESIGN.md reading R5), output popcount and the per-cycle trace of sampled words.
// The last block to finish advances the device cycle counter.
constexpr unsigned long long MISR_POLY = 0x42F0E1EBA9EA3693ULL;   // CRC-64/ECMA-182

__global__ void __launch_bounds__(256) k_end_cycle(EndArgs a, uint32_t latch_blocks) {
    pdl_entry();
    const unsigned long long c = a.ctl->cycle;
    if (blockIdx.x < latch_blocks) {
        // leftover latches (register D not fused into its gate's store): 16-byte copies,
        // grid-stride over (latch, vector)
        const uint32_t vpr = a.stride / 16;                         // stride is a multiple of 8
        if (vpr * 16 == a.stride) {
            const uint64_t n = (uint64_t)a.n_latch * vpr;
            for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n;
                 t += (uint64_t)latch_blocks * blockDim.x) {
                const uint32_t e = (uint32_t)(t / vpr), v = (uint32_t)(t - (uint64_t)e * vpr);
                const uint32_t src = resolve(__ldg(a.latch_src + e), a.qcur);
                const uint32_t dst = a.row_q0 + __ldg(a.latch_dst + e) + a.qnext;
                reinterpret_cast<uint4*>(a.state + (uint64_t)dst * a.stride)[v] =
                    __ldcs(reinterpret_cast<const uint4*>(a.state + (uint64_t)src * a.stride) + v);
            }
        } else {
            const uint64_t n = (uint64_t)a.n_latch * a.words;
            for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n;
                 t += (uint64_t)latch_blocks * blockDim.x) {
                const uint32_t e = (uint32_t)(t / a.words), w = (uint32_t)(t - (uint64_t)e * a.words);
                const uint32_t src = resolve(__ldg(a.latch_src + e), a.qcur);
                const uint32_t dst = a.row_q0 + __ldg(a.latch_dst + e) + a.qnext;
                reinterpret_cast<unsigned long long*>(a.state + (uint64_t)dst * a.stride)[w] =
                    reinterpret_cast<const unsigned long long*>(a.state + (uint64_t)src * a.stride)[w];
            }
        }
    } else {
        // thread = (bit-plane j, word w), consecutive threads = consecutive words, so every
        // PO row read is coalesced.  MISR planes are double-buffered by cycle parity: read
        // misr_cur (state after cycle c-1), write misr_next.
        const uint64_t t = (uint64_t)(blockIdx.x - latch_blocks) * blockDim.x + threadIdx.x;
        uint32_t pop = 0;
        if (t < (uint64_t)64 * a.words) {
            const uint32_t j = (uint32_t)(t / a.words), w = (uint32_t)(t - (uint64_t)j * a.words);
            const int32_t slot = (a.trace && c < a.trace_cap) ? __ldg(a.trace_slot + w) : -1;
            // full per-cycle output stream: a boolean, never a null pointer plus an offset
            const bool to_sink = a.ctl->sink_ptr && c - a.ctl->sink_base < a.ctl->sink_cycles;
            unsigned long long* sink = reinterpret_cast<unsigned long long*>(a.ctl->sink_ptr) +
                                       (to_sink ? (c - a.ctl->sink_base) * a.n_po * (uint64_t)a.words : 0ull);
            unsigned long long v = 0;
            for (uint32_t o = j; o < a.n_po; o += 64) {
                const uint32_t row = resolve(__ldg(a.po_rows + o), a.qcur);
                const unsigned long long x = __ldg(reinterpret_cast<const unsigned long long*>(a.state + (uint64_t)row * a.stride) + w);
                v ^= x;
                pop += __popcll(x);
                if (slot >= 0) a.trace[((uint64_t)c * a.n_po + o) * a.ntw + slot] = x;
                if (to_sink) sink[(uint64_t)o * a.words + w] = x;
            }
            const unsigned long long prev = j ? a.misr_cur[(uint64_t)(j - 1) * a.words + w] : 0ULL;
            const unsigned long long fb = ((MISR_POLY >> j) & 1ULL) ? a.misr_cur[(uint64_t)63 * a.words + w] : 0ULL;
            a.misr_next[(uint64_t)j * a.words + w] = prev ^ fb ^ v;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) pop += __shfl_xor_sync(FULL, pop, o);
        if ((threadIdx.x & 31) == 0 && pop) atomicAdd(&a.ctl->popcount, (unsigned long long)pop);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned int prev = atomicAdd(&a.ctl->done, 1u);
        if (prev == gridDim.x - 1) {
            a.ctl->done = 0u;
            a.ctl->cycle = c + 1;
            __threadfence();
        }
    }
}

cudaError_t launch_end_cycle(const EndArgs& a, cudaStream_t s) {
    // latch copies: grid-stride, at most ~8 blocks per SM worth of threads
    const uint64_t lt = (uint64_t)a.n_latch * (a.words > 1 ? a.words / 2 : 1);
    const uint32_t latch_blocks = (uint32_t)std::min<uint64_t>((lt + 255) / 256, 148 * 8);
    const uint32_t misr_blocks = (uint32_t)(((uint64_t)a.words * 64 + 255) / 256);
    return launch_k(k_end_cycle, latch_blocks + misr_blocks, s, a.pdl, a, latch_blocks);
}

// --------------------------------------------------------------------- utilities
// Rebinds the stimulus source and the output sink from kernel parameters (no host memory
// whose lifetime the asynchronous copy would depend on): gs_sim_run_streamed's chunks.
__global__ void k_set_binding(Ctl* ctl, unsigned long long stim_ptr, unsigned long long stim_base,
                              unsigned int stim_mode, unsigned long long sink_ptr, unsigned long long sink_base,
                              unsigned long long sink_cycles) {
    ctl->stim_ptr = stim_ptr;
    ctl->stim_base = stim_base;
    ctl->stim_mode = stim_mode;
    ctl->sink_ptr = sink_ptr;
    ctl->sink_base = sink_base;
    ctl->sink_cycles = sink_cycles;
}

cudaError_t launch_set_binding(Ctl* ctl, unsigned long long stim_ptr, unsigned long long stim_base,
                               unsigned int stim_mode, unsigned long long sink_ptr, unsigned long long sink_base,
                               unsigned long long sink_cycles, cudaStream_t s) {
    k_set_binding<<<1, 1, 0, s>>>(ctl, stim_ptr, stim_base, stim_mode, sink_ptr, sink_base, sink_cycles);
    return cudaGetLastError();
}

__global__ void k_fill_rows(uint8_t* state, uint64_t stride, uint32_t words, uint32_t row0, uint32_t nrows,
                            const uint8_t* init, int value) {
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (uint64_t)nrows * words) return;
    const uint32_t r = (uint32_t)(t / words), w = (uint32_t)(t - (uint64_t)r * words);
    const int bit = init ? init[r] : value;
    reinterpret_cast<unsigned long long*>(state + (uint64_t)(row0 + r) * stride)[w] = bit ? ~0ULL : 0ULL;
}

cudaError_t launch_fill_rows(uint8_t* state, uint64_t stride, uint32_t words, uint32_t row0, uint32_t nrows,
                             const uint8_t* init, int value, cudaStream_t s) {
    const uint64_t n = (uint64_t)nrows * words;
    if (n == 0) return cudaSuccess;
    k_fill_rows<<<(uint32_t)((n + 255) / 256), 256, 0, s>>>(state, stride, words, row0, nrows, init, value);
    return cudaGetLastError();
}

__global__ void k_gather_rows(const uint8_t* state, uint64_t stride, uint32_t words, const uint32_t* rows,
                              uint32_t n, uint32_t qcur, unsigned long long* out) {
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (uint64_t)n * words) return;
    const uint32_t o = (uint32_t)(t / words), w = (uint32_t)(t - (uint64_t)o * words);
    out[t] = reinterpret_cast<const unsigned long long*>(state + (uint64_t)resolve(rows[o], qcur) * stride)[w];
}

cudaError_t launch_gather_rows(const uint8_t* state, uint64_t stride, uint32_t words, const uint32_t* rows,
                               uint32_t n, uint32_t qcur, unsigned long long* out, cudaStream_t s) {
    const uint64_t t = (uint64_t)n * words;
    if (t == 0) return cudaSuccess;
    k_gather_rows<<<(uint32_t)((t + 255) / 256), 256, 0, s>>>(state, stride, words, rows, n, qcur, out);
    return cudaGetLastError();
}

// per-lane signature: transpose the 64 bit-planes of the lane's word (R5), then the
// job signature term mix64(sig ^ mix64(global lane)) summed mod 2^64 (R6).
__global__ void __launch_bounds__(256) k_lane_sigs(Ctl* ctl, const unsigned long long* misr, uint32_t words,
                                                   uint64_t lane_offset, unsigned long long* lane_sigs) {
    const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    unsigned long long term = 0;
    if (s < (uint64_t)words * 64) {
        const uint32_t w = (uint32_t)(s >> 6), b = (uint32_t)(s & 63);
        unsigned long long sig = 0;
        for (int j = 0; j < 64; ++j) sig |= ((misr[(uint64_t)j * words + w] >> b) & 1ULL) << j;
        lane_sigs[s] = sig;
        term = dmix64(sig ^ dmix64(lane_offset + s));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) term += __shfl_xor_sync(FULL, term, o);
    if ((threadIdx.x & 31) == 0 && term) atomicAdd(&ctl->sig_sum, term);
}

cudaError_t launch_lane_sigs(Ctl* ctl, const unsigned long long* misr, uint32_t words, uint64_t lane_offset,
                             unsigned long long* lane_sigs, cudaStream_t s) {
    const uint64_t n = (uint64_t)words * 64;
    if (n == 0) return cudaSuccess;
    k_lane_sigs<<<(uint32_t)((n + 255) / 256), 256, 0, s>>>(ctl, misr, words, lane_offset, lane_sigs);
    return cudaGetLastError();
}

}  // namespace gs
