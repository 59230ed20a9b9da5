// kernels_cluster.cu — kernel C: cluster-persistent levelized evaluation (sm_100a).
//
// Kernel A runs one launch per level over every lane of the batch, so (i) every level pays a
// launch boundary (ramp, drain, launch latency: C3 spends ~3 us per level) and (ii) the rows a
// level writes are re-read by the next level only after a whole level's worth of traffic for
// EVERY lane has gone through L2 (C4: 128 MB per level vs 126 MB of L2), so most gate-input
// reads go to DRAM.
//
// Kernel C keeps the same state layout and per-gate evaluation as kernel A but changes the
// schedule.  Lanes are independent, so the batch is cut into lane SLABS (a few
// 16-byte vectors of every row); a thread-block CLUSTER owns one slab at a time and walks
// every level of every cycle of a gs_sim_step for it, the cluster's CTAs splitting each
// level's gates between them, with a hardware cluster barrier (barrier.cluster arrive.release
// / wait.acquire) between levels instead of a launch boundary.  Slabs come from an atomic
// queue (Ctl::tile_next).  Only the clusters' slabs are in flight, so the rows a level writes
// are still in L2 when the next levels read them; the slab width and cluster size are chosen
// so that the lanes in flight fit the working set in L2 (gs_sim_opts.slab_lanes /
// cluster_size).  State rows are read with ld.global.cg (L2; written by other CTAs of the
// cluster during the launch), descriptors through the read-only path.
//
// Per cycle of a slab (same semantics as kernel A + k_stim + k_end_cycle, bit-identical):
//   PI rows of the slab (counter hash R2 or the bound buffer) -> barrier ->
//   every non-empty level (gates, fused latch into the other Q bank) -> barrier after each ->
//   leftover latches, MISR planes (R5), popcount, trace, output sink -> barrier.
#include <algorithm>

#include <cuda_runtime.h>

#include "device.cuh"
#include "kernels.h"

namespace gs {

#ifndef GS_CLUSTER_CTA
#define GS_CLUSTER_CTA 256
#endif
#ifndef GS_CLUSTER_MINB
#define GS_CLUSTER_MINB 4
#endif
constexpr uint32_t CLUSTER_CTA = GS_CLUSTER_CTA;   // threads per CTA (several CTAs per SM)
constexpr unsigned long long C_MISR_POLY = 0x42F0E1EBA9EA3693ULL;   // CRC-64/ECMA-182

__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n"
                 "barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_ncta() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
// read a 32-bit word of CTA `rank`'s shared memory (DSMEM)
__device__ __forceinline__ uint32_t ld_dsmem_u32(const void* local, uint32_t rank) {
    uint32_t addr = (uint32_t)__cvta_generic_to_shared(local), remote, v;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(addr), "r"(rank));
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(remote) : "memory");
    return v;
}

__device__ __forceinline__ uint4 ldcg4(const uint8_t* state, uint64_t stride, uint32_t row, uint32_t vec) {
    return __ldcg(reinterpret_cast<const uint4*>(state + (uint64_t)row * stride) + vec);
}

// One gate on VPT 16-byte vectors (vec, vec + VG, ...) of the slab: all VPT*k loads issued
// before use, one descriptor decode.
template <int K, int VPT>
__device__ __forceinline__ void c_gate(const ClusterArgs& a, uint32_t gate, const uint4& in, uint64_t tt,
                                       uint32_t qdst, uint32_t vec, uint32_t vg, uint32_t qcur, uint32_t qnext) {
    uint32_t r[8];
    r[0] = in.x; r[1] = in.y; r[2] = in.z; r[3] = in.w;
    if (K > 4) {
        const uint4 hi = __ldg(a.dhi + gate);
        r[4] = hi.x; r[5] = hi.y; r[6] = hi.z; r[7] = hi.w;
    }
    uint32_t row[K];
#pragma unroll
    for (int i = 0; i < K; ++i) row[i] = resolve(r[i], qcur);
    uint4* dst = reinterpret_cast<uint4*>(a.state + (uint64_t)(a.row_gate0 + gate) * a.stride);
    const bool latch = qdst != 0xFFFFFFFFu;
    uint4* qd = reinterpret_cast<uint4*>(a.state + (uint64_t)((latch ? qdst : 0u) + qnext) * a.stride);
    if constexpr (K <= 6) {
        uint4 x[VPT][K];
#pragma unroll
        for (int u = 0; u < VPT; ++u)
#pragma unroll
            for (int i = 0; i < K; ++i) x[u][i] = ldcg4(a.state, a.stride, row[i], vec + u * vg);
#pragma unroll
        for (int u = 0; u < VPT; ++u) {
            const uint4 y = lut_eval4<K>(tt, x[u]);
            dst[vec + u * vg] = y;
            if (latch) qd[vec + u * vg] = y;
        }
    } else {
        const uint4 t01 = __ldg(a.dtt + 2 * (uint64_t)gate), t23 = __ldg(a.dtt + 2 * (uint64_t)gate + 1);
        const uint64_t t4[4] = {((uint64_t)t01.y << 32) | t01.x, ((uint64_t)t01.w << 32) | t01.z,
                                ((uint64_t)t23.y << 32) | t23.x, ((uint64_t)t23.w << 32) | t23.z};
#pragma unroll 1
        for (int u = 0; u < VPT; ++u) {
            uint4 x[K];
#pragma unroll
            for (int i = 0; i < K; ++i) x[i] = ldcg4(a.state, a.stride, row[i], vec + u * vg);
            uint4 y;
            uint32_t* yp = reinterpret_cast<uint32_t*>(&y);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                uint32_t xs[K];
#pragma unroll
                for (int i = 0; i < K; ++i) xs[i] = reinterpret_cast<const uint32_t*>(&x[i])[j];
                yp[j] = lut_eval_big<K>(t4, xs);
            }
            dst[vec + u * vg] = y;
            if (latch) qd[vec + u * vg] = y;
        }
    }
}

template <int VPT>
__global__ void __launch_bounds__(CLUSTER_CTA, GS_CLUSTER_MINB) k_cluster(ClusterArgs a) {
    __shared__ uint32_t s_slab;
    const uint32_t rank = cluster_rank(), ncta = cluster_ncta();
    const uint32_t gtid = rank * blockDim.x + threadIdx.x, gtot = ncta * blockDim.x;
    // loop-invariant control state, read once
    const unsigned long long c0 = a.ctl->cycle;
    const unsigned long long seed = a.ctl->seed;
    const uint32_t stim_mode = a.ctl->stim_mode;
    const unsigned long long* stim_src = reinterpret_cast<const unsigned long long*>(a.ctl->stim_ptr);
    const unsigned long long stim_base = a.ctl->stim_base;
    const unsigned long long sink_ptr = a.ctl->sink_ptr, sink_base = a.ctl->sink_base,
                             sink_cycles = a.ctl->sink_cycles;
    const uint32_t SV = a.slab_vec;                  // 16-byte vectors per slab row
    const uint32_t SW = SV * 2;                      // 64-bit words per slab row
    const uint32_t VG = SV / VPT;                    // threads per gate (a power of two)
    const uint32_t vgs = 31u - __clz(VG);
    unsigned long long pop = 0;
    for (;;) {
        // ---- next slab of the cluster: CTA 0 claims it, every CTA reads it over DSMEM
        if (rank == 0 && threadIdx.x == 0) s_slab = atomicAdd(a.tile_next, 1u);
        cluster_sync_all();
        const uint32_t slab = ld_dsmem_u32(&s_slab, 0);
        if (slab >= a.n_slabs) {
            cluster_sync_all();                      // CTA 0's shared memory outlives every read
            break;
        }
        const uint32_t w0 = slab * SW, v0 = slab * SV;   // first word / vector of the slab
        for (uint32_t c = 0; c < a.ncycles; ++c) {
            const unsigned long long cyc = c0 + c;
            const uint32_t par = (uint32_t)(cyc & 1);
            const uint32_t qcur = par ? a.n_reg : 0u, qnext = par ? 0u : a.n_reg;
            // ---- primary inputs of this cycle (R2)
            for (uint32_t u = gtid; u < a.n_pi * SW; u += gtot) {
                const uint32_t p = u / SW, w = w0 + (u - p * SW);
                const unsigned long long v =
                    stim_mode == 0 ? dmix64(dmix64(dmix64(seed ^ p) ^ cyc) ^ (a.word_off + w))
                                   : stim_src[((cyc - stim_base) * a.n_pi + p) * a.words + w];
                reinterpret_cast<unsigned long long*>(a.state + (uint64_t)(a.row_pi0 + p) * a.stride)[w] = v;
            }
            cluster_sync_all();
            // ---- levels: (gate, vector group) units of the slab over the whole cluster
#pragma unroll 1
            for (uint32_t si = 0; si < a.n_steps; ++si) {
                const uint2 st = __ldg(a.steps + si);
                const uint32_t n = (st.y & STEP_N_MASK) * VG;
#pragma unroll 1
                for (uint32_t u = gtid; u < n; u += gtot) {
                    const uint32_t gi = u >> vgs, vgi = u & (VG - 1);
                    const uint32_t gate = st.x + gi;
                    const uint4 in = __ldg(a.din + gate);
                    const uint4 au = __ldg(reinterpret_cast<const uint4*>(a.aux) + gate);
                    const uint64_t tt = ((uint64_t)au.y << 32) | au.x;
                    const uint32_t qdst = au.z, vec = v0 + vgi;
                    switch (au.w & 0xFFu) {
                        case 1: c_gate<1, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        case 2: c_gate<2, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        case 3: c_gate<3, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        case 4: c_gate<4, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        case 5: c_gate<5, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        case 6: c_gate<6, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        case 7: c_gate<7, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                        default: c_gate<8, VPT>(a, gate, in, tt, qdst, vec, VG, qcur, qnext); break;
                    }
                }
                cluster_sync_all();
            }
            // ---- leftover latches (other Q bank) and the output MISR / popcount / trace / sink
            for (uint32_t u = gtid; u < a.n_latch * SV; u += gtot) {
                const uint32_t e = u / SV, v = v0 + (u - e * SV);
                const uint32_t src = resolve(__ldg(a.latch_src + e), qcur);
                const uint32_t dst = a.row_q0 + __ldg(a.latch_dst + e) + qnext;
                reinterpret_cast<uint4*>(a.state + (uint64_t)dst * a.stride)[v] = ldcg4(a.state, a.stride, src, v);
            }
            const unsigned long long* misr_cur = a.misr + (size_t)par * 64 * a.words;
            unsigned long long* misr_next = a.misr + (size_t)(par ^ 1) * 64 * a.words;
            const int32_t tr = (a.trace && cyc < a.trace_cap) ? 1 : 0;
            const bool to_sink = sink_ptr && cyc - sink_base < sink_cycles;
            unsigned long long* sink = reinterpret_cast<unsigned long long*>(sink_ptr) +
                                       (to_sink ? (cyc - sink_base) * a.n_po * (uint64_t)a.words : 0ull);
            for (uint32_t u = gtid; u < 64 * SW; u += gtot) {
                const uint32_t j = u / SW, w = w0 + (u - j * SW);
                const int32_t slot = tr ? __ldg(a.trace_slot + w) : -1;
                unsigned long long v = 0;
                for (uint32_t o = j; o < a.n_po; o += 64) {
                    const uint32_t row = resolve(__ldg(a.po_rows + o), qcur);
                    const unsigned long long x =
                        __ldcg(reinterpret_cast<const unsigned long long*>(a.state + (uint64_t)row * a.stride) + w);
                    v ^= x;
                    pop += __popcll(x);
                    if (slot >= 0) a.trace[((uint64_t)cyc * a.n_po + o) * a.ntw + slot] = x;
                    if (to_sink) sink[(uint64_t)o * a.words + w] = x;
                }
                const unsigned long long prev = j ? __ldcg(misr_cur + (uint64_t)(j - 1) * a.words + w) : 0ULL;
                const unsigned long long fb =
                    ((C_MISR_POLY >> j) & 1ULL) ? __ldcg(misr_cur + (uint64_t)63 * a.words + w) : 0ULL;
                misr_next[(uint64_t)j * a.words + w] = prev ^ fb ^ v;
            }
            cluster_sync_all();
        }
    }
    // ---- counters; the last CTA advances the device clock
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) pop += __shfl_xor_sync(FULL, pop, o);
    if ((threadIdx.x & 31) == 0 && pop) atomicAdd(&a.ctl->popcount, pop);
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned int prev = atomicAdd(&a.ctl->done, 1u);
        if (prev == gridDim.x - 1) {
            a.ctl->done = 0u;
            a.ctl->cycle = c0 + a.ncycles;
            __threadfence();
        }
    }
}

template <int VPT>
static cudaError_t cluster_launch_vpt(const ClusterArgs& a, uint32_t clusters, uint32_t cs, cudaStream_t s) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(clusters * cs);
    cfg.blockDim = dim3(CLUSTER_CTA);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cs;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_cluster<VPT>, a);
}

template <int VPT>
static cudaError_t cluster_occupancy_vpt(uint32_t cs, int* clusters) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(cs * 64);
    cfg.blockDim = dim3(CLUSTER_CTA);
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cs;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (cs > 8) {
        cudaError_t e = cudaFuncSetAttribute(k_cluster<VPT>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
    }
    return cudaOccupancyMaxActiveClusters(clusters, k_cluster<VPT>, &cfg);
}

uint32_t cluster_vpt(uint32_t slab_vec) { return slab_vec % 2 == 0 ? 2u : 1u; }   // VPT must divide the slab

cudaError_t cluster_max_active(uint32_t slab_vec, uint32_t cs, uint32_t* clusters) {
    int n = 0;
    cudaError_t e = cluster_vpt(slab_vec) == 2 ? cluster_occupancy_vpt<2>(cs, &n) : cluster_occupancy_vpt<1>(cs, &n);
    *clusters = e == cudaSuccess && n > 0 ? (uint32_t)n : 0u;
    return e;
}

cudaError_t launch_cluster(const ClusterArgs& a, uint32_t clusters, uint32_t cs, cudaStream_t s) {
    if (a.n_slabs == 0 || a.ncycles == 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(a.tile_next, 0, sizeof(unsigned int), s);   // empty the slab queue
    if (e != cudaSuccess) return e;
    return cluster_vpt(a.slab_vec) == 2 ? cluster_launch_vpt<2>(a, clusters, cs, s)
                                        : cluster_launch_vpt<1>(a, clusters, cs, s);
}

}  // namespace gs
