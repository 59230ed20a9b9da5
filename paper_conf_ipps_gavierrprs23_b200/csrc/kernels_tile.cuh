// kernels_tile.cuh — kernel T: tile-resident simulation in shared memory (sm_100a).
// Template definitions; instantiated per tile width in kernels_tile_tw{4,8,16,32,64}.cu
// (parallel compilation), dispatched by kernels_tile.cu.
//
// Stimuli are independent, so a tile of 32*TW lanes can run every level of
// every cycle of a step without ever synchronising with another tile.  One CTA owns a
// tile at a time: its live state (slots of tile.cpp: constants, PIs, both register
// banks, gate values by live range) sits in shared memory as TW 32-bit words per slot,
// and each level (one merged NN layer) is one pass of the CTA over
// (gate, word) units separated by __syncthreads.  HBM sees only the register rows and
// MISR planes at the start and end of a step: no per-level launch, no per-level round
// trip through HBM.  Narrow, deep circuits (the 32x32 multiplier has 184 levels of median
// width 28) are latency-bound per tile, so many tiles run per SM at once.
//
// Semantics are exactly kernel A's: the same PI hash (R2), the same double-buffered
// latch (R3), outputs sampled before the latch (R4), the same bit-sliced MISR (R5), so
// lane signatures, outputs, registers and the trace are bit-identical.
#pragma once

#include <type_traits>

#include <cuda_runtime.h>

#include "device.cuh"
#include "kernels.h"

namespace gs {

constexpr uint32_t TILE_CTA = 512;                   // threads per CTA (one CTA per SM)
#ifndef GS_TILE_VPT
#define GS_TILE_VPT 2
#endif
constexpr uint32_t TILE_VPT = GS_TILE_VPT;          // 16-byte vectors per thread and gate (TW >= 16)
constexpr unsigned long long TILE_MISR_POLY = 0x42F0E1EBA9EA3693ULL;   // CRC-64/ECMA-182
constexpr uint32_t TILE_CHUNK = GS_TILE_CHUNK;      // TMA-streamed descriptors per step (max)

// ---- TMA bulk copy (cp.async.bulk) of a level's descriptors into shared memory, completion
// signalled on an mbarrier (expect_tx / complete_tx), consumers wait on the phase parity
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
// dst_s / bar_s: shared-memory addresses (precomputed, see mbar_wait)
__device__ __forceinline__ void tma_load_1d(uint32_t dst_s, const void* src, uint32_t bytes, uint32_t bar_s) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // prior generic reads of dst
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar_s), "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(dst_s), "l"(src), "r"(bytes), "r"(bar_s)
                 : "memory");
}
// bar_s: the mbarrier's shared-memory address (computed once per kernel: the generic-to-
// shared conversion costs an S2R of the CTA id, which sat on every level's critical path)
__device__ __forceinline__ void mbar_wait(uint32_t bar_s, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(bar_s), "r"(parity), "r"(1000000u)   // suspend (<= 1 ms), not spin
            : "memory");
    }
}

// One gate on P 16-byte groups (4 words = 128 lanes each, VS uint4 apart) of its slots:
// the descriptor is decoded and the truth-table masks built once for the P vectors, and
// all P*K shared-memory loads are issued before the first is used.  HASQ: the circuit has
// registers (fused latch of the gate's value into the next register bank).
template <int K, bool HASQ, int P>
__device__ __forceinline__ void tile_gate(uint4* sl, uint32_t V, uint32_t v, uint32_t VS, const uint4& d,
                                          const uint4* desc_hi, uint32_t g, uint32_t q0, uint32_t qnext) {
    constexpr int KS = K > 4 ? 8 : 4;
    uint32_t s[KS];
    s[0] = d.x & 0xFFFFu; s[1] = d.x >> 16; s[2] = d.y & 0xFFFFu; s[3] = d.y >> 16;
    uint64_t t4[4] = {d.z & 0xFFFFu, 0, 0, 0};
    if (K > 4) {                                       // desc_hi[g] = {inputs 4..7, 256-bit table}
        const uint4 h0 = __ldg(desc_hi + 3 * (uint64_t)g), h1 = __ldg(desc_hi + 3 * (uint64_t)g + 1);
        s[4] = h0.x & 0xFFFFu; s[5] = h0.x >> 16; s[6] = h0.y & 0xFFFFu; s[7] = h0.y >> 16;
        t4[0] = ((uint64_t)h1.y << 32) | h1.x;
        t4[1] = ((uint64_t)h1.w << 32) | h1.z;
        if (K > 7) {
            const uint4 h2 = __ldg(desc_hi + 3 * (uint64_t)g + 2);
            t4[2] = ((uint64_t)h2.y << 32) | h2.x;
            t4[3] = ((uint64_t)h2.w << 32) | h2.z;
        }
    }
    uint4* dst = sl + (size_t)(d.z >> 16) * V + v;
    // fused latch: a boolean and an always-valid pointer (never null + offset)
    const uint32_t reg = HASQ ? d.w >> 4 : 0u;
    const bool latch = HASQ && reg != 0u;
    uint4* qd = sl + (size_t)(q0 + (latch ? reg - 1 : 0u) + qnext) * V + v;
    if constexpr (K <= 4) {
        const LutMasks<K> mk = lut_masks<K>(t4[0]);
        uint4 x[P][K];
#pragma unroll
        for (int p = 0; p < P; ++p)
#pragma unroll
            for (int i = 0; i < K; ++i) x[p][i] = sl[(size_t)s[i] * V + v + p * VS];
#pragma unroll
        for (int p = 0; p < P; ++p) {
            const uint4 y = lut_eval4_m<K>(mk, x[p]);
            dst[p * VS] = y;
            if (latch) qd[p * VS] = y;
        }
    } else {
#pragma unroll 1
        for (int p = 0; p < P; ++p) {
            uint4 x[K];
#pragma unroll
            for (int i = 0; i < K; ++i) x[i] = sl[(size_t)s[i] * V + v + p * VS];
            uint4 y;
            if (K <= 6) {
                y = lut_eval4<K <= 6 ? K : 6>(t4[0], x);
            } else {
                uint32_t xs[8];
                uint32_t* yp = reinterpret_cast<uint32_t*>(&y);
#pragma unroll
                for (int j = 0; j < 4; ++j) {
#pragma unroll
                    for (int i = 0; i < K; ++i) xs[i] = reinterpret_cast<const uint32_t*>(&x[i])[j];
                    yp[j] = lut_eval_big<K <= 6 ? 7 : K>(t4, xs);
                }
            }
            dst[p * VS] = y;
            if (latch) qd[p * VS] = y;
        }
    }
}

// a descriptor as the 16-byte form (narrow descriptors: inputs 0-1, table and output slot)
__device__ __forceinline__ uint4 as_desc4(const uint4& d) { return d; }
__device__ __forceinline__ uint4 as_desc4(const uint2& d) { return make_uint4(d.x, 0u, d.y, 0u); }

// All (gate, vector group) units of one step, every gate with fan-in K.
template <int K, bool HASQ, int P, uint32_t VS, uint32_t VSH, uint32_t GT, typename DT>
__device__ __forceinline__ void tile_step(uint4* sl, uint32_t V, const DT* dl, uint32_t g0, uint32_t n,
                                          uint32_t tid, const uint4* desc_hi, uint32_t q0, uint32_t R) {
#pragma unroll 1
    for (uint32_t u = tid; u < n; u += GT) {
        const uint32_t gi = u >> VSH, v = u & (VS - 1);
        tile_gate<K, HASQ, P>(sl, V, v, VS, as_desc4(dl[gi]), desc_hi, g0 + gi, q0, R);
    }
}

__device__ __forceinline__ void group_sync(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// TW = 32-bit words per slot (tile = 32 * TW lanes).  A thread evaluates one gate on P
// 16-byte groups of 4 words (128 lanes each; P = TILE_VPT when TW >= 16): P*k 16-byte
// shared-memory loads, P*4*(2^k - 1) LOP3, P 16-byte stores.  The CTA (TILE_CTA threads) is
// split into NG independent groups; each group simulates its own tile and synchronises only
// with itself (named barrier 1 + gid), so one group's level barrier overlaps the other
// groups' work.  Tiles are handed out by an atomic queue (Ctl::tile_next), one per group at a
// time.
//
// The level loop walks a per-program STEP table in shared memory: one step per non-empty
// level (resident descriptors), or per chunk of at most TILE_CHUNK gates of a level
// (TMA-streamed descriptors: chunk t+1 is copied into the other half of a fixed double
// buffer while chunk t is evaluated).  Every step ends with the group barrier.  Everything
// loop-invariant (Ctl fields, shared-memory addresses) is read once per launch, so a step
// costs a handful of instructions besides its gates.
template <int TW, bool HASQ, int NG, int DMN>
__global__ void __launch_bounds__(TILE_CTA, 1) k_tile(TileArgs a) {
    // DM: descriptor mode (0 global, 1 resident, 2 TMA-streamed chunks); DMN | 4: narrow 8-byte
    // descriptors (k <= 2, no registers)
    constexpr int DM = DMN & 3;
    constexpr bool NARROW = (DMN & 4) != 0;
    using DT = typename std::conditional<NARROW, uint2, uint4>::type;
    constexpr uint32_t V = TW / 4;                       // uint4 per slot
    constexpr uint32_t P = V >= 4 ? TILE_VPT : 1;        // 16-byte vectors per thread and gate
    constexpr uint32_t VS = V / P;                       // threads per gate (vector stride)
    constexpr uint32_t VSH = VS == 1 ? 0 : VS == 2 ? 1 : VS == 4 ? 2 : VS == 8 ? 3 : 4;
    static_assert((1u << VSH) == VS, "VS must be a power of two <= 16");
    constexpr uint32_t GT = TILE_CTA / NG;               // threads per group
    extern __shared__ uint4 smem[];
    // ---- shared layout: [resident descriptors (DM 1)] [steps: uint2 x n_steps, padded]
    //      then per group: [2 mbarriers (16 B)] [tile id (16 B)] [2 x TILE_CHUNK descriptors
    //                      (DM 2)] [slots: n_slots x V uint4] [MISR: 64 x V uint4]
    uint4* base = smem;
    if (DM == 1) {
        const DT* gd = reinterpret_cast<const DT*>(a.desc);
        DT* sd = reinterpret_cast<DT*>(smem);
        for (uint32_t i = threadIdx.x; i < a.n_eval; i += blockDim.x) sd[i] = __ldg(gd + i);
        base += ((size_t)a.n_eval * sizeof(DT) + 15) / 16;
    }
    uint2* steps = reinterpret_cast<uint2*>(base);
    for (uint32_t i = threadIdx.x; i < a.n_steps; i += blockDim.x) steps[i] = __ldg(a.steps + i);
    base += (a.n_steps + 1) / 2;
    const uint32_t gid = threadIdx.x / GT, tid = threadIdx.x % GT;
    const uint32_t bar = 1 + gid;
    uint4* greg = base + (size_t)gid * (2 + (DM == 2 ? 2 * TILE_CHUNK : 0) + (a.n_slots + 64) * V);
    uint64_t* mbar = reinterpret_cast<uint64_t*>(greg);
    volatile uint32_t* tile_slot = reinterpret_cast<volatile uint32_t*>(greg + 1);
    uint4* dbuf = greg + 2;                                   // DM 2: [2][TILE_CHUNK]
    uint4* sl = greg + 2 + (DM == 2 ? 2 * TILE_CHUNK : 0);    // slots
    const DT* dsm = DM == 1 ? reinterpret_cast<const DT*>(smem) : reinterpret_cast<const DT*>(a.desc);
    if (DM == 2 && tid == 0) {
        mbar_init(mbar, 1);
        mbar_init(mbar + 1, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const uint32_t mbar_s = smem_u32(mbar);
    const uint32_t dbuf_s = smem_u32(dbuf);
    uint32_t* sw = reinterpret_cast<uint32_t*>(sl);          // slots as 32-bit words
    uint32_t* mp = sw + (size_t)a.n_slots * TW;              // MISR planes [64][TW]
    // loop-invariant control state, read once
    const unsigned long long c0 = a.ctl->cycle;
    const unsigned long long seed = a.ctl->seed;
    const uint32_t stim_mode = a.ctl->stim_mode;
    const unsigned long long* stim_src = reinterpret_cast<const unsigned long long*>(a.ctl->stim_ptr);
    const unsigned long long stim_base = a.ctl->stim_base;
    const unsigned long long sink_ptr = a.ctl->sink_ptr, sink_base = a.ctl->sink_base,
                             sink_cycles = a.ctl->sink_cycles;
    const uint32_t R = a.n_reg, q0 = a.q0, n_steps = a.n_steps;
    const uint32_t w32_row = a.words * 2;                     // 32-bit words per state row
    const uint32_t* st32 = reinterpret_cast<const uint32_t*>(a.state);
    uint32_t* st32w = reinterpret_cast<uint32_t*>(a.state);
    // MISR planes are double-buffered by cycle parity (as k_end_cycle): read the buffer of
    // the first cycle, write the buffer of the cycle after the last
    const uint32_t* misr_in = reinterpret_cast<const uint32_t*>(a.misr + (size_t)(c0 & 1) * 64 * a.words);
    uint32_t* misr_out = reinterpret_cast<uint32_t*>(a.misr + (size_t)((c0 + a.ncycles) & 1) * 64 * a.words);
    unsigned long long pop = 0;
    uint32_t step = 0;                                        // DM 2: chunks consumed by this group

    // first tile of the group (the queue is zeroed before every launch)
    if (tid == 0) *tile_slot = atomicAdd(a.tile_next, 1u);
    group_sync(bar, GT);
    uint32_t tile = *tile_slot;
    group_sync(bar, GT);                                  // every thread has read it before the next claim
    if (DM == 2 && tid == 0 && tile < a.n_tiles && n_steps) {
        const uint2 s0 = steps[0];
        tma_load_1d(dbuf_s, reinterpret_cast<const DT*>(a.desc) + s0.x, (s0.y & STEP_N_MASK) * (uint32_t)sizeof(DT),
                    mbar_s);
    }
    while (tile < a.n_tiles) {
        // claim the next tile now, so the descriptor stream knows whether to continue
        if (tid == 0) *tile_slot = atomicAdd(a.tile_next, 1u);
        const uint32_t t0 = tile * TW;                    // first 32-bit word of the tile (shard-local)
        // ---- load: constants, both register banks, MISR planes
        for (uint32_t u = tid; u < TW; u += GT) {
            sw[u] = 0u;
            sw[TW + u] = 0xFFFFFFFFu;
        }
        // register slots: bank 0 always holds the CURRENT Q (state bank c0 & 1), bank 1 the
        // next one; inputs never resolve banks — bank 1 is copied into bank 0 after each cycle
        for (uint32_t u = tid; u < 2 * R * TW; u += GT) {
            const uint32_t r = u / TW, w = u % TW;
            const uint32_t sb = (r < R ? (uint32_t)(c0 & 1) : (uint32_t)((c0 + 1) & 1)) * R + (r < R ? r : r - R);
            sw[(size_t)(q0 + r) * TW + w] = st32[(uint64_t)(a.row_q0 + sb) * w32_row + t0 + w];
        }
        for (uint32_t u = tid; u < 64 * TW; u += GT) {
            const uint32_t j = u / TW, w = u % TW;
            mp[u] = misr_in[(uint64_t)j * w32_row + t0 + w];
        }
        group_sync(bar, GT);
        const uint32_t next_tile = *tile_slot;           // (written before the barrier above)
        for (uint32_t c = 0; c < a.ncycles; ++c) {
            const unsigned long long cyc = c0 + c;
            // ---- primary inputs of this cycle (R2): one 64-bit hash per pair of words
            for (uint32_t u = tid; u < a.n_pi * (TW / 2); u += GT) {
                const uint32_t p = u / (TW / 2), w2 = u % (TW / 2);
                const uint32_t g64 = (t0 >> 1) + w2;      // shard-local 64-bit word
                const unsigned long long v =
                    stim_mode == 0 ? dmix64(dmix64(dmix64(seed ^ p) ^ cyc) ^ (a.word_off + g64))
                                   : stim_src[((cyc - stim_base) * a.n_pi + p) * a.words + g64];
                reinterpret_cast<unsigned long long*>(sw + (size_t)(2 + p) * TW)[w2] = v;
            }
            group_sync(bar, GT);
            // ---- steps: every (gate, vector group) unit of the step, then the group barrier
            const bool more = c + 1 < a.ncycles || next_tile < a.n_tiles;   // stream continues
#pragma unroll 1
            for (uint32_t si = 0; si < n_steps; ++si) {
                const uint2 st = steps[si];
                const uint32_t sn_gates = st.y & STEP_N_MASK;
                const DT* dl = dsm + st.x;
                if (DM == 2) {
                    const uint32_t b = step & 1;
                    if (tid == 0 && (si + 1 < n_steps || more)) {
                        const uint2 sn = steps[si + 1 < n_steps ? si + 1 : 0];
                        tma_load_1d(dbuf_s + (b ^ 1) * (TILE_CHUNK * 16), reinterpret_cast<const DT*>(a.desc) + sn.x,
                                    (sn.y & STEP_N_MASK) * (uint32_t)sizeof(DT), mbar_s + 8 * (b ^ 1));
                    }
                    mbar_wait(mbar_s + 8 * b, (step >> 1) & 1);
                    dl = reinterpret_cast<const DT*>(dbuf + b * TILE_CHUNK);
                    ++step;
                }
                // every gate of a step has the same fan-in k (steps are cut at k changes), so the
                // dispatch happens once per step, not per gate
                const uint32_t n = sn_gates << VSH;
                switch ((st.y >> 24) & 15u) {
                    case 2: tile_step<2, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    case 3: tile_step<3, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    case 4: tile_step<4, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    case 1: tile_step<1, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    case 5: tile_step<5, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    case 6: tile_step<6, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    case 7: tile_step<7, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                    default: tile_step<8, HASQ, P, VS, VSH, GT>(sl, V, dl, st.x, n, tid, a.desc_hi, q0, R); break;
                }
                // the level barrier; TMA mode also needs it between the chunks of a level (the
                // next chunk's copy reuses the buffer the previous chunk was read from)
                if (DM == 2 || (st.y >> 31)) group_sync(bar, GT);
            }
            // ---- leftover latches into the next bank; MISR / popcount / trace of the POs
            for (uint32_t u = tid; u < a.n_latch * V; u += GT) {
                const uint32_t e = u / V, v = u % V;
                const uint32_t s = __ldg(a.latch_src + e);
                sl[(size_t)(q0 + __ldg(a.latch_dst + e) + R) * V + v] = sl[(size_t)s * V + v];
            }
            constexpr uint32_t NP = (64 * TW + GT - 1) / GT;    // MISR plane words per thread
            uint32_t newp[NP];
            const bool tr = a.trace && cyc < a.trace_cap;
            // full per-cycle output stream: a boolean, never a null pointer plus an offset
            const bool to_sink = sink_ptr && cyc - sink_base < sink_cycles;
            uint32_t* sink = reinterpret_cast<uint32_t*>(sink_ptr) +
                             (to_sink ? (cyc - sink_base) * a.n_po * (uint64_t)w32_row : 0ull);
#pragma unroll
            for (uint32_t i = 0; i < NP; ++i) {
                const uint32_t u = tid + i * GT;
                newp[i] = 0u;
                if (u < 64 * TW) {
                    const uint32_t j = u / TW, w = u % TW;
                    const uint32_t g32 = t0 + w;
                    const int32_t tslot = tr ? __ldg(a.trace_slot + (g32 >> 1)) : -1;
                    uint32_t vv = 0;
                    for (uint32_t o = j; o < a.n_po; o += 64) {
                        const uint32_t x = sw[(size_t)__ldg(a.po_slot + o) * TW + w];
                        vv ^= x;
                        pop += __popc(x);
                        if (tslot >= 0)
                            reinterpret_cast<uint32_t*>(a.trace)[(((uint64_t)cyc * a.n_po + o) * a.ntw + tslot) * 2 +
                                                                 (g32 & 1)] = x;
                        if (to_sink) sink[(uint64_t)o * w32_row + g32] = x;
                    }
                    const uint32_t prev = j ? mp[(j - 1) * TW + w] : 0u;
                    const uint32_t fb = ((TILE_MISR_POLY >> j) & 1ULL) ? mp[63 * TW + w] : 0u;
                    newp[i] = prev ^ fb ^ vv;
                }
            }
            group_sync(bar, GT);
#pragma unroll
            for (uint32_t i = 0; i < NP; ++i)
                if (tid + i * GT < 64 * TW) mp[tid + i * GT] = newp[i];
            if (HASQ && c + 1 < a.ncycles)                    // the clock edge: Q := next Q
                for (uint32_t u = tid; u < R * V; u += GT) sl[(size_t)q0 * V + u] = sl[(size_t)(q0 + R) * V + u];
            group_sync(bar, GT);
        }
        // ---- write back: Q of the last cycle (bank 0) to state bank (last & 1), the latched
        // next Q (bank 1) to the other bank; PO rows (read_outputs); MISR planes
        const uint32_t lastp = (uint32_t)((c0 + a.ncycles - 1) & 1);
        for (uint32_t u = tid; u < 2 * R * TW; u += GT) {
            const uint32_t r = u / TW, w = u % TW;
            const uint32_t sb = (r < R ? lastp : lastp ^ 1u) * R + (r < R ? r : r - R);
            st32w[(uint64_t)(a.row_q0 + sb) * w32_row + t0 + w] = sw[(size_t)(q0 + r) * TW + w];
        }
        for (uint32_t u = tid; u < a.n_wb * TW; u += GT) {
            const uint32_t e = u / TW, w = u % TW;
            st32w[(uint64_t)__ldg(a.wb_row + e) * w32_row + t0 + w] = sw[(size_t)__ldg(a.wb_slot + e) * TW + w];
        }
        for (uint32_t u = tid; u < 64 * TW; u += GT) {
            const uint32_t j = u / TW, w = u % TW;
            misr_out[(uint64_t)j * w32_row + t0 + w] = mp[u];
        }
        tile = next_tile;
        group_sync(bar, GT);                              // before the next tile reuses smem
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

// per-TW entry points (kernels_tile_tw*.cu)
template <int TW>
cudaError_t tile_setup_tw(uint32_t ng, size_t smem, int dm, bool has_q, int* per_sm);
template <int TW>
cudaError_t launch_tile_tw(const TileArgs& a, uint32_t ng, uint32_t grid, size_t smem, cudaStream_t s);

}  // namespace gs
