// device.cuh — device helpers shared by the sm_100a kernels (kernels.cu, kernels_tile.cu).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace gs {

#define FULL 0xFFFFFFFFu

__device__ __forceinline__ uint32_t resolve(uint32_t ref, uint32_t qcur) {
    // Q rows are referenced bank-0 relative with QFLAG; add the current bank offset
    return (ref & 0x7FFFFFFFu) + ((ref >> 31) ? qcur : 0u);
}

// ----------------------------------------------------------------------------- hash
// splitmix64 finaliser + the counter-based stimulus hash of DESIGN.md reading R2.
__device__ __forceinline__ unsigned long long dmix64(unsigned long long z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

// ------------------------------------------------------- programmatic dependent launch
// Every kernel of the per-cycle chain is launched with programmatic stream serialization
// (when enabled): it may become resident while its predecessor drains, and waits at
// griddepcontrol.wait until the predecessor has completed and its writes are visible.
// It immediately allows its own successor to launch.  Without the launch attribute both
// instructions are no-ops, so the kernels are correct either way.
__device__ __forceinline__ void pdl_entry() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// L1 prefetch of a line of program constants (gate descriptors), issued before pdl_entry()
// so its latency overlaps the previous kernel's drain
__device__ __forceinline__ void prefetch_l1(const void* p) {
    asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
}

template <typename... KArgs, typename... Args>
static cudaError_t launch_k(void (*kern)(KArgs...), uint32_t blocks, cudaStream_t s, uint32_t pdl,
                            Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = pdl ? at : nullptr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

// ------------------------------------------------------------------ kernel A: LUT
// Bit-sliced Shannon expansion of an LSB-first truth table: stage 0 selects between
// the minterm constants with x_0, stage i muxes pairs with x_i.  All operands are
// 32-bit so every mux is one LOP3.
template <int K>
__device__ __forceinline__ uint32_t lut_eval(uint64_t tt, const uint32_t* x);

// K = 5, 6: Shannon-expand on the top variables over 16-entry sub-tables, one at a
// time, so the register footprint stays that of K = 4 (keeps occupancy up).
template <int K>
__device__ __forceinline__ uint32_t lut_eval_wide(uint64_t tt, const uint32_t* x) {
    static_assert(K == 5 || K == 6, "lut_eval_wide: K = 5, 6");
    uint32_t y[4];
#pragma unroll 1
    for (int j = 0; j < (1 << (K - 4)); ++j) y[j] = lut_eval<4>(tt >> (16 * j), x);
    if (K == 5) return (x[4] & y[1]) | (~x[4] & y[0]);
    const uint32_t lo = (x[4] & y[1]) | (~x[4] & y[0]);
    const uint32_t hi = (x[4] & y[3]) | (~x[4] & y[2]);
    return (x[5] & hi) | (~x[5] & lo);
}

// s ? a : b bitwise, as ONE LOP3 (0xCA = F0 & CC | ~F0 & AA); written as PTX so the
// compiler cannot split it into SEL/NOT sequences
__device__ __forceinline__ uint32_t mux32(uint32_t s, uint32_t a, uint32_t b) {
    uint32_t d;
    asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(d) : "r"(s), "r"(a), "r"(b));
    return d;
}

// minterm masks of a K <= 4 table: m[i] = all-ones iff f(i) = 1 (bit i of tt, LSB-first);
// computed once per gate and shared by every word the thread evaluates
template <int K>
struct LutMasks {
    uint32_t m[1 << K];
};
template <int K>
__device__ __forceinline__ LutMasks<K> lut_masks(uint64_t tt) {
    LutMasks<K> r;
    const uint32_t t = (uint32_t)tt;                   // K <= 4: 16 table bits
#pragma unroll
    for (int i = 0; i < (1 << K); ++i)                 // sign-extended bit field: SHF + SGXT
        asm("bfe.s32 %0, %1, %2, 1;" : "=r"(r.m[i]) : "r"(t), "r"(i));
    return r;
}

// Shannon mux tree over the masks: 2^K - 1 LOP3 per 32 lanes
template <int K>
__device__ __forceinline__ uint32_t lut_eval_m(const LutMasks<K>& mk, const uint32_t* x) {
    if constexpr (K == 0) {
        return mk.m[0];
    } else {
        uint32_t v[1 << (K - 1)];
#pragma unroll
        for (int j = 0; j < (1 << (K - 1)); ++j) v[j] = mux32(x[0], mk.m[2 * j + 1], mk.m[2 * j]);
#pragma unroll
        for (int i = 1; i < K; ++i) {
#pragma unroll
            for (int j = 0; j < (1 << (K - 1 - i)); ++j) v[j] = mux32(x[i], v[2 * j + 1], v[2 * j]);
        }
        return v[0];
    }
}

template <int K>
__device__ __forceinline__ uint32_t lut_eval(uint64_t tt, const uint32_t* x) {
    if constexpr (K > 4) return lut_eval_wide<K>(tt, x);
    else return lut_eval_m<K>(lut_masks<K>(tt), x);
}


// K = 7, 8: Shannon expansion on x_6 (and x_7) over the 64-bit sub-tables t4[0..3] of the
// 2^K-bit table (2 x 63 + 1 or 4 x 63 + 3 LOP3 per 32 lanes)
template <int K>
__device__ __forceinline__ uint32_t lut_eval_big(const uint64_t* t4, const uint32_t* x) {
    const uint32_t y0 = lut_eval<6>(t4[0], x), y1 = lut_eval<6>(t4[1], x);
    const uint32_t lo = (x[6] & y1) | (~x[6] & y0);
    if (K == 7) return lo;
    const uint32_t y2 = lut_eval<6>(t4[2], x), y3 = lut_eval<6>(t4[3], x);
    const uint32_t hi = (x[6] & y3) | (~x[6] & y2);
    return (x[7] & hi) | (~x[7] & lo);
}

// evaluate one 16-byte vector (4 x 32 lanes) of a K <= 4 gate from precomputed masks
template <int K>
__device__ __forceinline__ uint4 lut_eval4_m(const LutMasks<K>& mk, const uint4* xv) {
    uint4 y;
    uint32_t x[K > 0 ? K : 1];
#pragma unroll
    for (int i = 0; i < K; ++i) x[i] = xv[i].x;
    y.x = lut_eval_m<K>(mk, x);
#pragma unroll
    for (int i = 0; i < K; ++i) x[i] = xv[i].y;
    y.y = lut_eval_m<K>(mk, x);
#pragma unroll
    for (int i = 0; i < K; ++i) x[i] = xv[i].z;
    y.z = lut_eval_m<K>(mk, x);
#pragma unroll
    for (int i = 0; i < K; ++i) x[i] = xv[i].w;
    y.w = lut_eval_m<K>(mk, x);
    return y;
}

// evaluate 4 x 32-bit lanes-words (one 16-byte vector) of a K-input gate
template <int K>
__device__ __forceinline__ uint4 lut_eval4(uint64_t tt, const uint4* xv) {
    if constexpr (K <= 4) return lut_eval4_m<K>(lut_masks<K>(tt), xv);
    else {
        uint4 y;
        uint32_t x[K];
#pragma unroll
        for (int i = 0; i < K; ++i) x[i] = xv[i].x;
        y.x = lut_eval<K>(tt, x);
#pragma unroll
        for (int i = 0; i < K; ++i) x[i] = xv[i].y;
        y.y = lut_eval<K>(tt, x);
#pragma unroll
        for (int i = 0; i < K; ++i) x[i] = xv[i].z;
        y.z = lut_eval<K>(tt, x);
#pragma unroll
        for (int i = 0; i < K; ++i) x[i] = xv[i].w;
        y.w = lut_eval<K>(tt, x);
        return y;
    }
}

}  // namespace gs
