// kernels.h — launch wrappers of the sm_100a kernels (kernels.cu).  Internal.
#pragma once

#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#include "internal.h"

namespace gs {

constexpr uint32_t GS_TILE_CHUNK = 256;   // kernel T: most descriptors per TMA-streamed step

// Device control block (first 256 B of the workspace).
struct Ctl {
    unsigned long long cycle;        // cycles stepped since reset (device-side clock)
    unsigned long long seed;         // generated-stimulus seed
    unsigned long long stim_ptr;     // host/device-bound stimulus [cycle][pi][word]
    unsigned long long stim_base;    // cycle index of stim_ptr's first cycle
    unsigned long long popcount;     // ones over all outputs of all cycles
    unsigned long long ab_mismatch;  // kernel B != kernel A (GS_KERNEL_AB)
    unsigned long long violations;   // kernel B outputs outside {0,1}
    unsigned long long sig_sum;      // scratch for gs_sim_read_signature
    unsigned int stim_mode;          // 0 generated, 1 bound buffer
    unsigned int done;               // last-block counter of the end-of-cycle kernel
    unsigned long long sink_ptr;     // 0, or device [cycle - sink_base][po][word] every output
    unsigned long long sink_base;    //   of every cycle is written to (gs_sim_run_streamed)
    unsigned long long sink_cycles;  //   capacity in cycles
    unsigned int tile_next;          // kernel T: next tile of the launch's queue (zeroed per launch)
    unsigned int pad_;
};

struct LevelArgs {
    const uint4* din;
    const GateAux* aux;
    const uint4* dhi;                 // inputs 4..7 (gates with k > 4)
    const uint4* dtt;                 // [n_eval][2] full 256-bit tables (programs with k > 6)
    const uint32_t* term_off;
    const uint32_t* terms;
    uint32_t g0, ng;                  // exec-order gate range of the level
    uint8_t* state;
    uint64_t stride;                  // bytes per state row (= lanes / 8)
    uint32_t words;                   // 64-bit words per row
    uint32_t row_gate0;
    uint32_t qcur, qnext;             // bank offsets (0 or n_reg) for Q refs / latch stores
    Ctl* ctl;
    uint32_t vec0, vslab;             // lane group in 16-byte vectors (vslab 0 = whole row)
    uint32_t unroll;                  // max vectors per thread on the wide path (0 = auto)
    uint32_t pdl;                     // launch with programmatic stream serialization
    uint32_t min_warps;               // auto U: prefer smaller U below this many warps
    uint32_t grid_blocks;             // wide path: cap the grid at the resident capacity (0 = off)
    uint32_t sms;                     // multiprocessors of the device
};

struct EndArgs {
    Ctl* ctl;
    uint8_t* state;
    uint64_t stride;
    uint32_t words;
    const uint32_t* latch_src;
    const uint32_t* latch_dst;
    uint32_t n_latch;
    uint32_t row_q0, qcur, qnext;
    const uint32_t* po_rows;
    uint32_t n_po;
    const unsigned long long* misr_cur;   // [64][words] MISR after the previous cycle
    unsigned long long* misr_next;        // [64][words] MISR after this cycle
    const int32_t* trace_slot;        // [words]
    unsigned long long* trace;        // [trace_cap][n_po][ntw]
    uint32_t ntw, trace_cap;
    uint32_t pdl;
};

// Kernel T (kernels_tile.cu): one lane tile per CTA at a time, all levels x all cycles of
// a step in shared memory (slots of tile.cpp); descriptors resident in shared memory
// when they fit.
struct TileArgs {
    const TileDesc* desc;             // [n_eval]
    const uint4* desc_hi;             // [n_eval] (k > 4 only)
    const uint2* steps;               // [n_steps] {first gate, gates}: one per non-empty level
                                      // (chunks of <= TILE_CHUNK gates when TMA-streamed)
    uint32_t n_eval, n_steps;
    uint32_t desc_smem;               // 0: descriptors read from global; 1: resident in shared
                                      // memory; 2: TMA-streamed step by step (double buffer);
                                      // | 4: narrow 8-byte descriptors (desc points at them)
    const uint32_t* po_slot;
    uint32_t n_po;
    const uint32_t* latch_src;
    const uint32_t* latch_dst;
    uint32_t n_latch;
    const uint32_t* wb_row;
    const uint32_t* wb_slot;
    uint32_t n_wb;
    uint32_t n_pi, n_reg, q0, n_slots;
    uint8_t* state;
    uint32_t words;                   // 64-bit words per state row (lanes / 64)
    uint32_t row_q0;
    Ctl* ctl;
    unsigned int* tile_next;          // &ctl->tile_next (the tile queue)
    unsigned long long* misr;         // 2 x [64][words] (buffer = cycle parity)
    const int32_t* trace_slot;
    unsigned long long* trace;
    uint32_t ntw, trace_cap;
    uint64_t word_off;                // global 64-bit word of local lane 0
    uint32_t ncycles, n_tiles;
};
// Steps of a program for kernels T and C: {first gate, n | k << 24 | level_end << 31}.  One
// step per run of equal fan-in k inside a non-empty level (aux != NULL; k = 0 when aux is
// NULL: one step per level), runs longer than `chunk` gates cut (chunk = 0: no cutting);
// level_end marks the last step of a level (the level barrier follows it).
constexpr uint32_t STEP_N_MASK = 0xFFFFFFu;
void tile_steps(const uint32_t* level_off, uint32_t n_levels, const GateAux* aux, uint32_t chunk,
                std::vector<uint2>& out);
size_t tile_smem_bytes(uint32_t tw, uint32_t ng, uint32_t n_slots, uint32_t n_eval, uint32_t n_steps,
                       int desc_mode);   // desc_mode | 4: narrow descriptors
cudaError_t tile_setup(uint32_t tw, uint32_t ng, uint32_t n_slots, uint32_t n_eval, uint32_t n_steps,
                       int desc_smem, uint32_t has_q, uint32_t* per_sm);
cudaError_t launch_tile(const TileArgs& a, uint32_t tw, uint32_t ng, uint32_t grid, cudaStream_t s);

// *grid_stride (may be NULL): bit 0 set when the launch's grid was capped at the resident
// capacity (the grid-stride branch), bit 1 when its warp units hold several gates
// Kernel C (kernels_cluster.cu): a thread-block cluster owns a lane slab and walks every
// level of every cycle of a step for it, cluster barrier between levels.
struct ClusterArgs {
    const uint4* din;
    const GateAux* aux;
    const uint4* dhi;                 // inputs 4..7 (gates with k > 4)
    const uint4* dtt;                 // [n_eval][2] full 256-bit tables (programs with k > 6)
    const uint2* steps;               // [n_steps] {first gate, gates} of every non-empty level
    uint32_t n_steps;
    uint8_t* state;
    uint64_t stride;                  // bytes per state row
    uint32_t words;                   // 64-bit words per row
    uint32_t row_gate0, row_pi0, n_pi, row_q0, n_reg;
    const uint32_t* latch_src;
    const uint32_t* latch_dst;
    uint32_t n_latch;
    const uint32_t* po_rows;
    uint32_t n_po;
    unsigned long long* misr;         // 2 x [64][words] (buffer = cycle parity)
    const int32_t* trace_slot;        // [words]
    unsigned long long* trace;
    uint32_t ntw, trace_cap;
    Ctl* ctl;
    unsigned int* tile_next;          // &ctl->tile_next (the slab queue)
    uint64_t word_off;                // global 64-bit word of local lane 0
    uint32_t ncycles;
    uint32_t slab_vec, n_slabs;       // 16-byte vectors per slab row; slabs = lanes / (128 slab_vec)
};
uint32_t cluster_vpt(uint32_t slab_vec);
cudaError_t cluster_max_active(uint32_t slab_vec, uint32_t cs, uint32_t* clusters);
cudaError_t launch_cluster(const ClusterArgs& a, uint32_t clusters, uint32_t cs, cudaStream_t s);

cudaError_t launch_level_lut(const LevelArgs& a, cudaStream_t s, uint32_t* grid_stride = nullptr);
uint32_t level_lut_resident_blocks(int device);   // CTAs of k_level_lut_wide resident on the GPU
cudaError_t launch_level_poly(const LevelArgs& a, int check_only, cudaStream_t s);
cudaError_t launch_stim(Ctl* ctl, uint8_t* state, uint64_t stride, uint32_t words, uint32_t row_pi0,
                        uint32_t n_pi, uint64_t word_off, uint32_t pdl, cudaStream_t s);
cudaError_t launch_end_cycle(const EndArgs& a, cudaStream_t s);
cudaError_t launch_set_binding(Ctl* ctl, unsigned long long stim_ptr, unsigned long long stim_base,
                               unsigned int stim_mode, unsigned long long sink_ptr, unsigned long long sink_base,
                               unsigned long long sink_cycles, cudaStream_t s);
cudaError_t launch_fill_rows(uint8_t* state, uint64_t stride, uint32_t words, uint32_t row0, uint32_t nrows,
                             const uint8_t* init, int value, cudaStream_t s);
cudaError_t launch_gather_rows(const uint8_t* state, uint64_t stride, uint32_t words, const uint32_t* rows,
                               uint32_t n, uint32_t qcur, unsigned long long* out, cudaStream_t s);
cudaError_t launch_lane_sigs(Ctl* ctl, const unsigned long long* misr, uint32_t words, uint64_t lane_offset,
                             unsigned long long* lane_sigs, cudaStream_t s);

}  // namespace gs
