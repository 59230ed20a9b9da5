/*
 * gsim.h — C-ABI of the B200-native batched, levelized circuit simulator.
 *
 * The calls follow the statement of the problem in PAPER.md (Gavier et al.,
 * "Neural Network Compiler for Parallel High-Throughput Simulation of Digital
 * Circuits"); "P:N" is PAPER.md line N.
 *
 *   netlist  : a digital circuit f:{0,1}^n -> {0,1}^m (§II-B) split into
 *              LUTs of at most L inputs forming a DAG (§III-B1), with
 *              D flip-flops on one global clock cut into pseudo-inputs
 *              (Q) and pseudo-outputs (D) joined by a recurrent connection
 *              (§III-C).
 *   compile  : levelize the DAG (the merged NN layers, §III-D) with
 *              level balancing, and compile every truth table to the
 *              coefficients of its multilinear polynomial (Eq. 1 P:115,
 *              Algorithm 1).
 *   simulate : bind a batch of stimuli, step N clock cycles on the GPU, read the
 *              outputs and register state back ("transfer the binary inputs
 *              ... binary outputs obtained"); verify by comparing outputs.
 *
 * Conventions (all calls):
 *   - Every call returns gs_status; GS_OK == 0, errors are negative.  The
 *     thread-local message of the last failure is gs_last_error().  No C++
 *     exception ever crosses this boundary.
 *   - Arrays passed in are COPIED; the library never keeps a caller pointer.
 *   - Device memory is CALLER-OWNED: the simulator works in one caller-provided
 *     device workspace (e.g. a torch uint8 CUDA tensor) sized by
 *     gs_sim_workspace_bytes; the hot path (gs_sim_step) never allocates.
 *     The single exception is gs_sim_bind_stimulus_host, which keeps a
 *     library-owned device staging buffer (grown on demand, freed by
 *     gs_sim_destroy) for the paper-style host->device stimulus transfer.
 *   - Handles are freed by their _destroy call; a gs_program must outlive every
 *     gs_sim created from it.  One gs_sim is used from one host thread / stream.
 *   - Lane s of a word is bit (s mod 64) of uint64 word floor(s/64) (little-endian:
 *     also correct when the same memory is viewed as 32-bit words).
 */
#ifndef GSIM_H
#define GSIM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GSIM_VERSION "0.2.0"
#define GS_MAX_K 6        /* largest fan-in of gs_add_gate (the table fits one uint64)        */
#define GS_MAX_K_POLY 8   /* largest LUT fan-in L of the netlist, the compiler and every kernel
                             ("4, 6 or 8"); tables of up to 2^8 bits (gs_add_gate_wide) */

typedef int32_t gs_status;
enum {
    GS_OK = 0,
    GS_ERR_ARG = -1,              /* bad argument / net id / truth-table bits >= 2^k   */
    GS_ERR_ARITY = -2,            /* k > GS_MAX_K (or > opts.max_k)                    */
    GS_ERR_UNDRIVEN = -3,         /* a register without D (gs_set_register_d)          */
    GS_ERR_COMB_LOOP = -4,        /* the gate graph is not a DAG (reading R8)   */
    GS_ERR_BUFFER_TOO_SMALL = -5, /* required size written back where documented       */
    GS_ERR_CUDA = -6,             /* a CUDA runtime error (message in gs_last_error)   */
    GS_ERR_STATE = -7,            /* call not valid in the current state               */
    GS_ERR_NOMEM = -8             /* host allocation failure                           */
};

typedef uint32_t gs_net;          /* net id; see the numbering rules below */
typedef struct gs_netlist gs_netlist;
typedef struct gs_program gs_program;
typedef struct gs_sim gs_sim;

/* Thread-local text of the last error (never NULL; "" after success). */
const char* gs_last_error(void);
const char* gs_version(void);
/* Build identity of the loaded library: a hash of every source file and compiler flag it was
 * built from (set by the in-tree build).  Measurement files keyed by it (profiles/traffic.json)
 * are refused by bench.py when the kernels changed since they were captured. */
const char* gs_build_id(void);

/* ======================================================================= netlist
 * Nets are numbered in creation order by the incremental calls.  Every add_*
 * call returns the new net id in *out.  A gate may reference any existing or
 * later net (the compiler sorts); the gate graph must be acyclic once registers
 * are cut (Q is a source, D a sink).
 */
gs_status gs_netlist_create(gs_netlist** out);
gs_status gs_netlist_destroy(gs_netlist* nl);

/* New primary input.  PIs are numbered 0,1,... in creation order (the "pi"
 * index used by stimulus layouts). */
gs_status gs_add_input(gs_netlist* nl, gs_net* out);

/* Constant net (a 0-input LUT, "LUTs smaller than L"); value must be 0 or 1. */
gs_status gs_add_const(gs_netlist* nl, int value, gs_net* out);

/* k-input LUT (0 <= k <= GS_MAX_K).  in[0..k-1] are net ids (repeats are
 * legal, reading R9).  tt is the truth table LSB-first: bit m = f(x) where x_i =
 * bit i of m (reading R1; the paper's Algorithm 1 nests x_1 outermost, which is
 * the same table under k-bit index reversal).  Bits >= 2^k must be zero. */
gs_status gs_add_gate(gs_netlist* nl, uint32_t k, const gs_net* in, uint64_t tt, gs_net* out);

/* Same for 0 <= k <= GS_MAX_K_POLY: tt_words holds the table LSB-first in max(1, 2^k / 64)
 * uint64 words (bit m of the table = bit m % 64 of word m / 64). */
gs_status gs_add_gate_wide(gs_netlist* nl, uint32_t k, const gs_net* in, const uint64_t* tt_words, gs_net* out);

/* D flip-flop on the global clock.  *q_out is its Q net (pseudo-input);
 * init (0/1) is Q at cycle 0 (reading R3).  Registers are numbered 0,1,... in
 * creation order (the "reg" index of register read/write layouts). */
gs_status gs_add_register(gs_netlist* nl, int init, gs_net* q_out);

/* Connect D of register q to net d (pseudo-output); separate from
 * creation so that feedback through registers can be built.  Re-setting is
 * allowed (last call wins). */
gs_status gs_set_register_d(gs_netlist* nl, gs_net q, gs_net d);

/* Mark net as a primary output; *po_index (may be NULL) receives its output
 * index (0,1,... in call order).  A net may be marked more than once. */
gs_status gs_mark_output(gs_netlist* nl, gs_net net, uint32_t* po_index);

/* Bulk load (10M-gate netlists).  Only valid on an EMPTY netlist.  Net ids:
 *   [0, n_pi)                  primary inputs 0..n_pi-1
 *   [n_pi, n_pi+n_reg)         register Q nets 0..n_reg-1
 *   [n_pi+n_reg, +n_gates)     gate g output
 * gate g has k = gate_k[g] inputs gate_in[gate_in_off[g] .. gate_in_off[g+1]),
 * truth table gate_tt[g]; register r has init reg_init[r] and D = reg_d[r];
 * outputs are po[0..n_po).  Same validity rules as the incremental calls. */
typedef struct {
    uint32_t n_pi, n_reg, n_gates, n_po;
    const uint8_t* reg_init;      /* [n_reg]     0/1                         */
    const uint32_t* reg_d;        /* [n_reg]     net ids                     */
    const uint8_t* gate_k;        /* [n_gates]                               */
    const uint32_t* gate_in_off;  /* [n_gates+1] CSR offsets, gate_in_off[0]=0 */
    const uint32_t* gate_in;      /* [gate_in_off[n_gates]] net ids          */
    const uint64_t* gate_tt;      /* [n_gates]   LSB-first truth tables (bits 0..63) */
    const uint32_t* po;           /* [n_po]      net ids                     */
    const uint64_t* gate_tt_hi;   /* [n_gates][3] table bits 64..255 of gates with k = 7, 8;
                                     may be NULL when no gate has k > 6            */
} gs_netlist_arrays;
gs_status gs_netlist_load_arrays(gs_netlist* nl, const gs_netlist_arrays* a);

typedef struct {
    uint32_t n_nets, n_pi, n_reg, n_gates, n_po;
    uint64_t n_edges;
} gs_netlist_counts;
gs_status gs_netlist_get_counts(const gs_netlist* nl, gs_netlist_counts* out);

/* ======================================================================= compile */
typedef struct {
    int balance;      /* 0: ASAP levels.  1: slack-based balancing within [ASAP, ALAP]
                         (same depth; flattens the unbalanced level widths).
                         2: ALAP levels (same depth; shortest live ranges, so the fewest
                         kernel-T shared-memory slots).  Results never depend on it.   */
    uint32_t max_k;   /* reject gates wider than this (0 = GS_MAX_K_POLY)             */
    uint32_t lut_k;   /* 0: evaluate the netlist's LUTs as given.  L in [2, max_k]: first
                         collapse cones into LUTs of at most L inputs (the paper's LUT
                         mapping step and its main hyperparameter L):
                         a gate absorbs its deepest gate input while the merged input set
                         has <= L nets (logic is duplicated where a cone is shared); gates
                         nobody reads any more report k = 0.  Same simulation results,
                         fewer levels and LUTs.                                        */
    uint64_t level_seed;  /* 0: levels from `balance`.  Otherwise every gate gets a seeded
                         RANDOM level in [1 + max level of its gate inputs, ALAP] (a valid
                         assignment of the same depth; results must not depend on it, a
                         property test of DESIGN.md reading R11).                      */
} gs_compile_opts;

/* Validate (GS_ERR_UNDRIVEN, GS_ERR_COMB_LOOP, GS_ERR_ARITY), optionally collapse cones
 * into <= lut_k-input LUTs, levelize (level(g) =
 * 1 + max level of its gate inputs; PIs, Qs, constants are level 0; optional
 * balancing), compile every TT to multilinear coefficients, lay out state rows and
 * pack per-level device descriptors.  opts may be NULL (balance=1). */
gs_status gs_compile(const gs_netlist* nl, const gs_compile_opts* opts, gs_program** out);
gs_status gs_program_destroy(gs_program* prog);

typedef struct {
    uint32_t n_pi, n_reg, n_po;
    uint32_t n_gates;          /* all gates of the netlist                               */
    uint32_t n_eval_gates;     /* gates evaluated per cycle (k >= 1) = G of the metric   */
    uint32_t n_levels;         /* depth D = number of merged NN layers           */
    uint32_t max_width, min_width;
    uint32_t k_hist[GS_MAX_K_POLY + 1];
    uint64_t n_edges;          /* sum of k over evaluated gates                          */
    uint64_t nnz_coeffs;       /* nonzero w_S over all gates ("connections" of the merged
                                  hidden->output layer)                    */
    uint64_t hidden_neurons;   /* sum 2^k (worst-case hidden neurons)             */
    uint64_t n_rows;           /* state rows                */
    uint64_t program_hash;     /* hash of the compiled program (multi-rank consistency)  */
} gs_program_info;
gs_status gs_program_get_info(const gs_program* prog, gs_program_info* out);

/* widths[l] = gates on level l+1 (l < n_levels).  n must be >= n_levels. */
gs_status gs_program_level_widths(const gs_program* prog, uint32_t* widths, uint32_t n);

/* level[g] for every gate in netlist order (0 for constants).  n >= n_gates. */
gs_status gs_program_gate_levels(const gs_program* prog, uint32_t* level, uint32_t n);

/* Multilinear coefficients w_S (LSB-first subset index) of gate g (netlist order),
 * as compiled by the Möbius butterfly (Algorithm 1 in iterative form).  n >= 2^k. */
gs_status gs_program_coeffs(const gs_program* prog, uint32_t gate, int32_t* w, uint32_t n);

/* The LUT the program evaluates for netlist gate `gate` (after optional cone collapsing):
 * its fan-in *k, input nets in[0..k-1] (in must hold GS_MAX_K_POLY entries) and the
 * LSB-first truth table in tt[0..3] (4 words; words past max(1, 2^k / 64) are zero).
 * Without lut_k this is the gate as added; absorbed gates report k = 0. */
gs_status gs_program_gate_lut(const gs_program* prog, uint32_t gate, uint32_t* k, gs_net* in, uint64_t* tt);

/* Persist / restore a compiled program (the paper's saved network model, Fig. 1):
 * a binary file of every table the simulator uses plus the query tables.  Loading checks the
 * format, a checksum, every table size, every index (row references in range and from an
 * earlier level, register / output / latch maps, term and coefficient offsets monotonic and
 * inside their arrays) and the program hash, and returns GS_ERR_ARG on a foreign, truncated,
 * edited or inconsistent file.  The loaded program behaves exactly like the one saved (same
 * program_hash). */
gs_status gs_program_save(const gs_program* prog, const char* path);
gs_status gs_program_load(const char* path, gs_program** out);

/* Shared-memory slots one lane tile of kernel T needs (constants, PIs, two register banks,
 * gate values reused by live range; tile.cpp).  A tile of 32*w lanes needs
 * (slots + 64) * 4 * w bytes of shared memory (<= 227 KB). */
gs_status gs_program_tile_slots(const gs_program* prog, uint32_t* slots);

/* ======================================================================= simulate */
enum {
    GS_KERNEL_AUTO = 0,   /* GS_KERNEL_TILE when every LUT has k <= 5, one tile's live
                             state fits shared memory next to the gate descriptors
                             (resident or TMA-streamed) and the levels average <= 400
                             gates (or lanes < 32,768); else GS_KERNEL_LUT               */
    GS_KERNEL_LUT = 1,    /* kernel A: bit-sliced LUT evaluation, 64 stimuli per word      */
    GS_KERNEL_POLY = 2,   /* kernel B: the paper's network (Eq. 1-3, Fig. 2) in exact
                             integer arithmetic, bit-sliced: per nonzero monomial S
                             the hidden neuron Theta(sum_{s in S} x_s - |S| + 1) as a
                             bit-plane counter, the output neuron sum_S w_S h_S as a
                             two's-complement bit-plane accumulator; outputs outside {0,1}
                             are counted                                            */
    GS_KERNEL_AB = 3,     /* A writes, B recomputes every level and counts mismatches      */
    /* 4: retired in 0.2.0 (an experimental persistent schedule, measured slower than A)   */
    GS_KERNEL_TILE = 5,    /* kernel T: each CTA owns a tile of 32*tile_words lanes and runs
                             every level of every cycle of a gs_sim_step in shared memory
                             (gate values in slots reused by live range); one launch per
                             step, HBM touched only for registers/MISR at step boundaries.
                             Needs the live slots of one tile to fit shared memory.          */
    GS_KERNEL_CLUSTER = 6  /* kernel C: kernel A's state layout and gate evaluation, but a
                             thread-block cluster owns a lane slab (slab_lanes lanes) and walks
                             every level of every cycle of a gs_sim_step for it, the cluster's
                             CTAs splitting each level, a hardware cluster barrier between
                             levels; slabs from an atomic queue.  One launch per step; the
                             lanes in flight are bounded so a level's rows are still in L2
                             when the next levels read them.                               */
};

typedef struct {
    int device;                   /* CUDA device ordinal                                   */
    void* stream;                 /* cudaStream_t all work is queued on (NULL = legacy)    */
    uint64_t lanes;               /* stimuli in this shard, multiple of 64                 */
    uint64_t lane_offset;         /* global index of local lane 0, multiple of 64          */
    int kernel;                   /* GS_KERNEL_*                                           */
    uint32_t n_trace_words;       /* local words whose outputs are recorded every cycle    */
    const uint32_t* trace_words;  /* [n_trace_words] local word indices (copied)           */
    uint32_t trace_cycles;        /* capacity of the trace, in cycles                      */
    int use_graphs;               /* 1: replay each cycle as a CUDA graph (default)        */
    uint32_t lut_unroll;          /* kernel A: max 16-byte vectors per thread (0 = auto)   */
    uint32_t flags;               /* GS_SIM_* bits below                                   */
    uint32_t tile_words;          /* TILE: 32-bit words per slot, lanes per tile = 32 * this
                                     (4, 8, 16, 32 or 64; 0 = auto); lanes % (32 * it) == 0 */
    uint32_t tile_groups;         /* TILE: independent thread groups (tiles) per 512-thread
                                     CTA, each with its own barrier (1, 2 or 4; 0 = auto)  */
    uint32_t lane_groups;         /* LUT: cut the lanes into this many groups whose level
                                     chains run CONCURRENTLY every cycle (parallel branches of
                                     the cycle's CUDA graph / streams), so one group's level
                                     ramp and drain overlap another's levels.  Needs
                                     (lanes/128) % groups == 0 and a multiple of 4096 lanes
                                     per group.  0 = auto, 1 = off.           */
    uint32_t cluster_size;        /* CLUSTER: CTAs per thread-block cluster (1, 2, 4, 8 or 16;
                                     0 = auto)                                             */
    uint32_t slab_lanes;          /* CLUSTER: lanes per slab, a multiple of 128 dividing lanes
                                     (0 = auto).
                                     LUT: lanes per slab of the segmented schedule (0 = off):
                                     every run of consecutive levels at least slab_min_gates
                                     wide executes slab after slab, each slab through all
                                     levels of the run, so a level's rows of the slab are
                                     still in L2 when the run's next levels read them; the
                                     other levels run over all lanes (of the lane group:
                                     each concurrent group runs its own slab schedule).  A
                                     multiple of 4096 dividing the lanes of a group; with
                                     lane_groups 0 the schedule runs as one group.         */
    uint32_t slab_min_gates;      /* LUT segmented schedule: narrowest level that runs per
                                     slab (0 = 32768 gates)                                */
} gs_sim_opts;
/* flags: launch the per-cycle kernels WITHOUT programmatic dependent launch (by default a
 * level kernel may become resident while its predecessor drains; A/B measurement only). */
#define GS_SIM_NO_PDL 1u
/* flags: kernel A launches one CTA per work chunk instead of a grid-stride grid sized to
 * the resident capacity (A/B measurement only). */
#define GS_SIM_NO_GRID_STRIDE 8u
/* flags (kernel T): force the descriptor source — global memory (L1/L2), a TMA bulk-copy
 * stream of <= 256 descriptors per step into a shared-memory double buffer, or the whole
 * table resident in shared memory.  Default: the planner's choice (sim.cpp make_plans). */
#define GS_SIM_TILE_DESC_GLOBAL 16u
#define GS_SIM_TILE_DESC_TMA 32u
#define GS_SIM_TILE_DESC_RESIDENT 512u   /* force the resident table (A/B measurement)        */
/* Retired in 0.2.0 (measured slower, DESIGN.md §6 "removed"): flag bits 2, 4 (L2 eviction
 * hints), 64, 128 (bulk-copy gathers) and 256 (kernel T slots in global memory) are rejected
 * with GS_ERR_ARG. */

/* Device workspace bytes required for (prog, opts). */
gs_status gs_sim_workspace_bytes(const gs_program* prog, const gs_sim_opts* opts, size_t* bytes);

/* Create a simulator in the caller's device workspace (256-byte aligned, >= the
 * size above, else GS_ERR_BUFFER_TOO_SMALL).  Uploads the program, then resets. */
gs_status gs_sim_create(const gs_program* prog, const gs_sim_opts* opts, void* dev_workspace,
                        size_t workspace_bytes, gs_sim** out);
gs_status gs_sim_destroy(gs_sim* sim);

/* Stimulus binding.  Generated: PI p of global lane s at cycle c is bit
 * (s mod 64) of H(seed, p, c, s/64), the counter-based hash of reading R2
 * (computed on the device every cycle; identical across shards).  Host: words
 * laid out [cycle][pi][local word], `cycles` cycles starting at the NEXT cycle
 * stepped; copied host->device on the stream (pinned memory recommended).
 * Device: the same layout already in caller-owned device memory (not copied;
 * must stay valid while stepping). */
gs_status gs_sim_bind_stimulus_generated(gs_sim* sim, uint64_t seed);
gs_status gs_sim_bind_stimulus_host(gs_sim* sim, const uint64_t* words, uint32_t cycles);
gs_status gs_sim_bind_stimulus_device(gs_sim* sim, const uint64_t* dev_words, uint32_t cycles);

/* Q := init, cycle := 0, MISR := 0, counters := 0, trace cleared. */
gs_status gs_sim_reset(gs_sim* sim);

/* Re-target the sim at another lane range of the same job: lane_offset := the new
 * global index of local lane 0 (a multiple of 64, else GS_ERR_ARG), then gs_sim_reset.
 * Stimuli are independent, so a batch larger than one GPU's memory runs as
 * sequential sub-batches in one workspace (C5 at fewer than 8 GPUs).
 * Synchronises the sim's stream; the cycle graphs are re-captured on the next step. */
gs_status gs_sim_set_lane_offset(gs_sim* sim, uint64_t lane_offset);

/* Advance ncycles clock cycles (asynchronous on the stream).  Per cycle: stimulus
 * rows, every level in order (gates + fused register latch into the other Q bank),
 * remaining latches, output MISR/trace.  GS_ERR_STATE if no stimulus is bound or a
 * host/device stimulus would run past its bound cycles. */
gs_status gs_sim_step(gs_sim* sim, uint32_t ncycles);
gs_status gs_sim_sync(gs_sim* sim);

/* Paper-style streamed run (the binary inputs are transferred to the GPU and the
 * binary outputs read back, inside the timed region): step `ncycles` cycles with stimuli
 * taken from host_stim [ncycles][n_pi][W] and EVERY output of EVERY cycle written to
 * host_out [ncycles][n_po][W] (NULL = no output stream), W = lanes/64.  Chunks of
 * `chunk` cycles (0 = 25) are pipelined: the host->device copy of chunk i+1 and the
 * device->host copy of chunk i-1 run on a library-owned copy stream while chunk i is
 * computed (pinned host buffers required for overlap).  Uses a library-owned device
 * staging buffer (2 x chunk of inputs and outputs, freed by gs_sim_destroy).  Asynchronous
 * on the sim's stream: host_out is complete after gs_sim_sync.  Afterwards a generated
 * binding that was in place before the call is restored; any other binding is cleared
 * (gs_sim_step returns GS_ERR_STATE until the caller binds again). */
gs_status gs_sim_run_streamed(gs_sim* sim, const uint64_t* host_stim, uint64_t* host_out, uint32_t ncycles,
                              uint32_t chunk);
gs_status gs_sim_get_cycle(const gs_sim* sim, uint64_t* cycle);
/* The resolved launch configuration: kernel (GS_KERNEL_*, AUTO resolved) and the number of
 * concurrent lane groups (1 = a single level chain per cycle). */
gs_status gs_sim_get_config(const gs_sim* sim, int* kernel, uint32_t* lane_groups);

/* The resolved launch plan of the sim (what gs_sim_step launches). */
typedef struct {
    int kernel;                   /* GS_KERNEL_* (AUTO resolved)                            */
    uint32_t lane_groups;         /* kernel A: concurrent lane groups                       */
    uint32_t tile_words, tile_groups, tile_desc;   /* kernel T: words per slot, thread groups
                                     per CTA, descriptor source (0 global, 1 resident, 2 TMA;
                                     | 4: narrow 8-byte descriptors, k <= 2 and no registers) */
    uint32_t grid;                /* kernels T / C: CTAs launched per step                  */
    uint32_t cluster_size, slab_lanes;             /* kernel C; slab_lanes also kernel A's slab
                                     schedule (0 = off)                                    */
    uint32_t live_slots;          /* kernel T: shared-memory slots per tile                 */
} gs_launch_info;
gs_status gs_sim_get_launch(const gs_sim* sim, gs_launch_info* out);

/* Readback (synchronous).  Layouts, with W = lanes/64 local words:
 *   outputs   [po][W]  outputs of the last stepped cycle (before its latch, R4)
 *   registers [reg][W] Q after the last clock edge
 *   trace     [cycle][po][n_trace_words] for the first trace_cycles cycles
 *   lane sigs [lanes]  per-lane 64-bit MISR over all outputs of all cycles (R5)
 * nwords is the capacity of the host buffer in uint64 (GS_ERR_BUFFER_TOO_SMALL). */
gs_status gs_sim_read_outputs(gs_sim* sim, uint64_t* host, size_t nwords);
gs_status gs_sim_read_registers(gs_sim* sim, uint64_t* host, size_t nwords);
gs_status gs_sim_write_registers(gs_sim* sim, const uint64_t* host, size_t nwords);
gs_status gs_sim_read_trace(gs_sim* sim, uint64_t* host, size_t nwords, uint32_t* cycles_recorded);
gs_status gs_sim_read_lane_signatures(gs_sim* sim, uint64_t* host, size_t nlanes);

typedef struct {
    uint64_t lane_sig_sum;          /* sum_s mix64(sig_s ^ mix64(s)) mod 2^64 (R6)     */
    uint64_t out_popcount;          /* ones over all outputs, lanes and cycles        */
    uint64_t ab_mismatch;           /* GS_KERNEL_AB: lane-cycles where B != A          */
    uint64_t invariant_violations;  /* kernel B outputs outside {0,1}         */
    uint64_t cycles;                /* cycles stepped since reset                     */
} gs_signature;
gs_status gs_sim_read_signature(gs_sim* sim, gs_signature* out);

/* Measurement support (bench.py roofline): step ncycles WITHOUT graphs, bracketing
 * every level launch with CUDA events on the sim's stream.  Writes the summed
 * device time of the level kernels, of the whole cycles, the number of level
 * launches and the algorithmic bytes the level kernels moved. */
typedef struct {
    double level_ms, total_ms;
    uint64_t level_launches, total_launches;
    double level_bytes;
    uint64_t grid_stride_launches;  /* kernel A level launches (host launch decisions; with lane
                                       groups one per captured graph) whose grid was capped at
                                       the resident CTA capacity, grid-striding over the level */
    uint64_t multi_gate_launches;   /* kernel A level launches (counted likewise) whose warp
                                       units hold several gates (rows < 16,384 lanes) */
} gs_profile;
gs_status gs_sim_profile_step(gs_sim* sim, uint32_t ncycles, gs_profile* out);

/* Number of kernel launches one gs_sim_step(1) issues (bench "gpu_launches"). */
gs_status gs_sim_launches_per_cycle(const gs_sim* sim, uint64_t* launches);

#ifdef __cplusplus
}
#endif
#endif /* GSIM_H */
