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
// Eq. 1-3) in exact integer arithmetic, bit-sliced over 64 stimuli per thread: hidden
// neuron h_S = Theta(sum_{s in S} x_s - |S| + 1) as a bit-plane counter, output
// sum_S w_S h_S (only the nonzero w_S, sparse as in P:187) as a two's-complement
// bit-plane accumulator.  Outputs outside {0,1} are counted (P:224 says they cannot
// happen).  Used standalone or as a cross-check of A.
#include <algorithm>

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
// U*k per thread, one descriptor fetch per U vectors).
template <int K, int U>
__device__ __forceinline__ void lut_gate_u(const LevelArgs& a, uint32_t gate, uint4 in, uint32_t v0,
                                           uint64_t tt, uint32_t qdst) {
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
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
        for (int i = 0; i < K; ++i) x[u][i] = __ldg(src[i] + u * 32);
    uint4* dst = reinterpret_cast<uint4*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride) + v0;
    // fused latch target: a boolean, never a null pointer plus an offset (the compiler may
    // assume such a pointer non-null and drop the test)
    const bool latch = qdst != 0xFFFFFFFFu;
    uint4* qd = reinterpret_cast<uint4*>(a.state + (uint64_t)((latch ? qdst : 0u) + a.qnext) * a.stride) + v0;
#pragma unroll
    for (int u = 0; u < U; ++u) {
        const uint4 y = lut_eval4<K>(tt, x[u]);
        dst[u * 32] = y;
        if (latch) qd[u * 32] = y;
    }
}

// One gate x U*32 vectors of any fan-in (the body of a kernel A warp unit).
template <int U>
__device__ __forceinline__ void lut_gate_any(const LevelArgs& a, uint32_t gate, uint4 in, uint4 au, uint32_t v0) {
    const uint64_t tt = ((uint64_t)au.y << 32) | au.x;
    const uint32_t qdst = au.z, k = au.w & 0xFFu;
    switch (k) {
        case 1: lut_gate_u<1, U>(a, gate, in, v0, tt, qdst); break;
        case 2: lut_gate_u<2, U>(a, gate, in, v0, tt, qdst); break;
        case 3: lut_gate_u<3, U>(a, gate, in, v0, tt, qdst); break;
        case 4: lut_gate_u<4, U>(a, gate, in, v0, tt, qdst); break;
        case 5: lut_gate_u<5, 1>(a, gate, in, v0, tt, qdst);
                if (U > 1) lut_gate_u<5, 1>(a, gate, in, v0 + 32, tt, qdst);
                if (U > 2) { lut_gate_u<5, 1>(a, gate, in, v0 + 64, tt, qdst);
                             lut_gate_u<5, 1>(a, gate, in, v0 + 96, tt, qdst); }
                if (U > 4)
                    for (int u = 4; u < U; ++u) lut_gate_u<5, 1>(a, gate, in, v0 + 32 * u, tt, qdst);
                break;
        case 6: lut_gate_u<6, 1>(a, gate, in, v0, tt, qdst);
                if (U > 1) lut_gate_u<6, 1>(a, gate, in, v0 + 32, tt, qdst);
                if (U > 2) { lut_gate_u<6, 1>(a, gate, in, v0 + 64, tt, qdst);
                             lut_gate_u<6, 1>(a, gate, in, v0 + 96, tt, qdst); }
                if (U > 4)
                    for (int u = 4; u < U; ++u) lut_gate_u<6, 1>(a, gate, in, v0 + 32 * u, tt, qdst);
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

// Grid-stride over warp units (gate, chunk of U*32 vectors): the grid is sized to the
// resident capacity (148 SMs x CTAs per SM, a.grid_blocks), so no level ends with a
// partially filled wave of CTAs.
#ifndef GS_U1_MINB
#define GS_U1_MINB 4
#endif
#ifndef GS_LUT_GP
#define GS_LUT_GP 1
#endif
#ifndef GS_GP_MINB
#define GS_GP_MINB 3
#endif
#ifndef GS_GP_VPT                 // gates x vectors per thread of a multi-gate warp unit
#define GS_GP_VPT 4
#endif
// PF (levels within one wave of resident CTAs, latency-bound launches): the first unit's
// descriptors -- program constants, independent of the previous level -- are prefetched into
// L1 before waiting for the previous level, so their latency overlaps its drain (C3 +3.5 %;
// on deep HBM-bound levels the extra registers cost ~1 %, so those launch without it)
template <int U, bool PF>
__global__ void __launch_bounds__(256, U > 4 ? 2 : U == 1 ? GS_U1_MINB : 4)
    k_level_lut_wide(LevelArgs a, uint32_t cpg_shift, uint32_t vec0) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t total = a.ng << cpg_shift;
    const uint32_t stride = (gridDim.x * blockDim.x) >> 5;
    const uint32_t warp0 = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (PF && warp0 < total && lane == 0) {
        prefetch_l1(a.din + a.g0 + (warp0 >> cpg_shift));
        prefetch_l1(a.aux + a.g0 + (warp0 >> cpg_shift));
    }
    pdl_entry();
    for (uint32_t warp = warp0; warp < total; warp += stride) {
        const uint32_t gi = warp >> cpg_shift;
        const uint32_t chunk = warp & ((1u << cpg_shift) - 1);
        const uint32_t gate = a.g0 + gi;
        lut_gate_any<U>(a, gate, __ldg(a.din + gate), __ldg(reinterpret_cast<const uint4*>(a.aux) + gate),
                        vec0 + chunk * 32 * U + lane);
    }
}

// Short rows (< 4 x 32 vectors per lane group, i.e. < 16,384 lanes): a warp unit is GP
// consecutive gates x U*32 vectors, with all GP*U*K input loads issued before any is used,
// so a thread keeps as many bytes in flight as on 2 KB rows (GP*U = 4).  Gates are k-grouped
// inside a level, so the GP gates share k except at a k-group edge (then one at a time).
template <int K, int U, int GP>
__device__ __forceinline__ void lut_gates_gp(const LevelArgs& a, uint32_t gate0, const uint4 (&in)[GP],
                                             const uint4 (&au)[GP], uint32_t v0) {
    uint4 x[GP][U][K];
#pragma unroll
    for (int g = 0; g < GP; ++g) {
        const uint32_t r[4] = {in[g].x, in[g].y, in[g].z, in[g].w};
#pragma unroll
        for (int i = 0; i < K; ++i) {
            const uint4* src = reinterpret_cast<const uint4*>(a.state + (uint64_t)resolve(r[i], a.qcur) * a.stride) + v0;
#pragma unroll
            for (int u = 0; u < U; ++u) x[g][u][i] = __ldg(src + u * 32);
        }
    }
#pragma unroll
    for (int g = 0; g < GP; ++g) {
        const uint64_t tt = ((uint64_t)au[g].y << 32) | au[g].x;
        const uint32_t qdst = au[g].z;
        uint4* dst = reinterpret_cast<uint4*>(a.state + (uint64_t)(a.row_gate0 + gate0 + g) * a.stride) + v0;
        const bool latch = qdst != 0xFFFFFFFFu;
        uint4* qd = reinterpret_cast<uint4*>(a.state + (uint64_t)((latch ? qdst : 0u) + a.qnext) * a.stride) + v0;
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint4 y = lut_eval4<K>(tt, x[g][u]);
            dst[u * 32] = y;
            if (latch) qd[u * 32] = y;
        }
    }
}

template <int U, int GP>
__global__ void __launch_bounds__(256, GS_GP_MINB) k_level_lut_gp(LevelArgs a, uint32_t cpg_shift, uint32_t vec0) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t total = ((a.ng + GP - 1) / GP) << cpg_shift;
    const uint32_t stride = (gridDim.x * blockDim.x) >> 5;
    pdl_entry();
    for (uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; warp < total; warp += stride) {
        const uint32_t gi0 = (warp >> cpg_shift) * GP;
        const uint32_t chunk = warp & ((1u << cpg_shift) - 1);
        const uint32_t v0 = vec0 + chunk * 32 * U + lane;
        const uint32_t n = min((uint32_t)GP, a.ng - gi0);
        const uint32_t gate0 = a.g0 + gi0;
        uint4 in[GP], au[GP];
#pragma unroll
        for (int g = 0; g < GP; ++g) {
            const uint32_t gate = gate0 + min((uint32_t)g, n - 1);
            in[g] = __ldg(a.din + gate);
            au[g] = __ldg(reinterpret_cast<const uint4*>(a.aux) + gate);
        }
        const uint32_t k = au[0].w & 0xFFu;
        bool uni = n == GP;
#pragma unroll
        for (int g = 1; g < GP; ++g) uni = uni && (au[g].w & 0xFFu) == k;
        if (uni && k >= 1 && k <= 4) {
            switch (k) {
                case 1: lut_gates_gp<1, U, GP>(a, gate0, in, au, v0); break;
                case 2: lut_gates_gp<2, U, GP>(a, gate0, in, au, v0); break;
                case 3: lut_gates_gp<3, U, GP>(a, gate0, in, au, v0); break;
                default: lut_gates_gp<4, U, GP>(a, gate0, in, au, v0); break;
            }
        } else {
#pragma unroll
            for (int g = 0; g < GP; ++g)
                if ((uint32_t)g < n) lut_gate_any<U>(a, gate0 + g, in[g], au[g], v0);
        }
    }
}

uint32_t level_lut_resident_blocks(int device) {
    int sms = 0, per = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) return 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_level_lut_wide<4, false>, 256, 0) != cudaSuccess)
        return 0;
    return (uint32_t)(sms * per);
}

cudaError_t launch_level_lut(const LevelArgs& a, cudaStream_t s, uint32_t* grid_stride) {
    if (grid_stride) *grid_stride = 0;
    if (a.ng == 0) return cudaSuccess;
    // lane group: 16-byte vectors [a.vec0, a.vec0 + a.vslab) of every row (whole row if vslab == 0)
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
            if (cap && blocks > cap && blocks <= 4 * cap) {
                blocks = cap;
                if (grid_stride) *grid_stride = 1;
            }
#if GS_LUT_GP
            // short rows: GP = 4 / U gates per warp unit when the level still fills a wave
            // of resident warps
            if (!a.unroll && U < 4 && cpg == 1) {
                const uint32_t GP = GS_GP_VPT / U;
                const uint64_t units = (uint64_t)((a.ng + GP - 1) / GP);
                const uint32_t gcap = a.grid_blocks / 4 * GS_GP_MINB;   // resident CTAs
                if (units >= (gcap ? (uint64_t)gcap * 8 : (uint64_t)a.min_warps)) {
                    uint32_t gblocks = (uint32_t)((units * 32 + 255) / 256);
                    if (grid_stride) *grid_stride = 0;
                    if (gcap && gblocks > gcap && gblocks <= 4 * gcap) {
                        gblocks = gcap;
                        if (grid_stride) *grid_stride = 1;
                    }
                    if (grid_stride) *grid_stride |= 2;
                    if (U == 2) return launch_k(k_level_lut_gp<2, GS_GP_VPT / 2>, gblocks, s, a.pdl, a, 0u, a.vec0);
                    return launch_k(k_level_lut_gp<1, GS_GP_VPT>, gblocks, s, a.pdl, a, 0u, a.vec0);
                }
            }
#endif
            if (cap && blocks <= cap) {      // one wave or less: prefetch the descriptors
                if (U == 8) return launch_k(k_level_lut_wide<8, true>, blocks, s, a.pdl, a, sh, a.vec0);
                if (U == 4) return launch_k(k_level_lut_wide<4, true>, blocks, s, a.pdl, a, sh, a.vec0);
                if (U == 2) return launch_k(k_level_lut_wide<2, true>, blocks, s, a.pdl, a, sh, a.vec0);
                return launch_k(k_level_lut_wide<1, true>, blocks, s, a.pdl, a, sh, a.vec0);
            }
            if (U == 8) return launch_k(k_level_lut_wide<8, false>, blocks, s, a.pdl, a, sh, a.vec0);
            if (U == 4) return launch_k(k_level_lut_wide<4, false>, blocks, s, a.pdl, a, sh, a.vec0);
            if (U == 2) return launch_k(k_level_lut_wide<2, false>, blocks, s, a.pdl, a, sh, a.vec0);
            return launch_k(k_level_lut_wide<1, false>, blocks, s, a.pdl, a, sh, a.vec0);
        }
    }
    if (a.vslab) return cudaErrorInvalidValue;      // lane groups only on the wide path
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
