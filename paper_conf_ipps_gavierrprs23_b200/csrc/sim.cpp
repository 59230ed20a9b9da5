// sim.cpp — the simulation engine half of the C-ABI (include/gsim.h).
//
// Per clock cycle (P:241 recurrent connection, P:271 stimulus in / outputs out):
//   stim kernel -> one level kernel per level (A, B or A+B) -> end-of-cycle kernel.
// The per-cycle launch sequence only depends on the Q-bank parity, so it is captured
// once per parity as a CUDA graph and replayed; the cycle index lives on the device
// (Ctl::cycle) and is advanced by the end-of-cycle kernel.
#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "internal.h"
#include "kernels.h"

using namespace gs;

namespace {

size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

struct Layout {
    size_t ctl, state, din, aux, dhi, dtt, term_off, terms, po_rows, latch_src, latch_dst, reg_init,
        trace_slot, misr, trace, lane_sigs, scratch, t_desc, t_desc_hi, t_po, t_lsrc, t_ldst, t_wbrow,
        t_wbslot, t_steps, total;
};

struct Plans {
    TilePlan tile;
    uint32_t tw = 0;                  // kernel T: 32-bit words per slot
    uint32_t ng = 0;                  // kernel T: thread groups (tiles) per CTA
    int desc_smem = 0;                // kernel T: descriptors 0 global, 1 resident, 2 TMA-streamed
                                      //   (| 4: narrow 8-byte descriptors)
    std::vector<uint2> steps;         // kernel T: level steps (chunks when TMA-streamed)
};

constexpr size_t TILE_SMEM_MAX = 232448;   // 227 KB opt-in shared memory per CTA (sm_100a)

gs_status make_plans(const Program& p, const gs_sim_opts& o, Plans& pl) {
    if (o.kernel == GS_KERNEL_CLUSTER) {
        const uint64_t sl = o.slab_lanes ? o.slab_lanes : 256;
        if (sl % 128 || o.lanes % sl || ((sl / 128) & (sl / 128 - 1)))
            return fail(GS_ERR_ARG, "CLUSTER: slab_lanes must be 128 x a power of two dividing lanes");
        const uint32_t cs = o.cluster_size ? o.cluster_size : 2;
        if (cs != 1 && cs != 2 && cs != 4 && cs != 8 && cs != 16)
            return fail(GS_ERR_ARG, "CLUSTER: cluster_size must be 1, 2, 4, 8 or 16");
        tile_steps(p.level_off.data(), p.n_levels, nullptr, 0, pl.steps);
        return GS_OK;
    }
    if (o.kernel != GS_KERNEL_TILE) return GS_OK;
    if (gs_status st = tile_plan(p, pl.tile)) return st;
    std::vector<uint2> st_level, st_chunk;
    tile_steps(p.level_off.data(), p.n_levels, p.aux.data(), 0, st_level);
    tile_steps(p.level_off.data(), p.n_levels, p.aux.data(), GS_TILE_CHUNK, st_chunk);
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, o.device);
    if (o.tile_words && (o.tile_words != 4 && o.tile_words != 8 && o.tile_words != 16 && o.tile_words != 32 &&
                         o.tile_words != 64))
        return fail(GS_ERR_ARG, "TILE: tile_words must be 4, 8, 16, 32 or 64");
    if (o.tile_groups && (o.tile_groups != 1 && o.tile_groups != 2 && o.tile_groups != 4))
        return fail(GS_ERR_ARG, "TILE: tile_groups must be 1, 2 or 4");
    if (o.tile_words && o.lanes % (32ull * o.tile_words))
        return fail(GS_ERR_ARG, "TILE: lanes must be a multiple of 32 * tile_words");
    // choose (descriptor mode, tile words, groups per CTA).  Kernel T is latency-bound per
    // tile (a level barrier per step), so a launch takes ~ waves x tile time with waves =
    // ceil(tiles / (groups x SMs)): score = lanes per wave (quantisation included) x a
    // descriptor-source weight, then more SMs busy, then wider tiles, then fewer groups.  C2 (256 live slots): 2 groups x 2,048-lane tiles with the
    // small descriptor table read through L1/L2, 3.18e13 (profiles/r02_kernelT_configs_C2.txt)
    const int forced = (o.flags & GS_SIM_TILE_DESC_GLOBAL) ? 0 : (o.flags & GS_SIM_TILE_DESC_TMA) ? 2
                       : (o.flags & GS_SIM_TILE_DESC_RESIDENT) ? 1 : -1;
    const bool narrow = !pl.tile.desc_n.empty();              // 8-byte descriptors (tile.cpp)
    const uint64_t table_bytes = (uint64_t)p.n_eval * (narrow ? 8 : 16);
    uint64_t best = 0;
    for (int ds : {1, 2, 0}) {
        if (forced >= 0 && ds != forced) continue;
        const uint32_t nsteps = (uint32_t)(ds == 2 ? st_chunk.size() : st_level.size());
        for (uint32_t ng : {4u, 2u, 1u}) {
            if (o.tile_groups && ng != o.tile_groups) continue;
            for (uint32_t tw : {4u, 8u, 16u, 32u, 64u}) {
                if (o.tile_words && tw != o.tile_words) continue;
                if (o.lanes % (32ull * tw)) continue;
                if (tile_smem_bytes(tw, ng, pl.tile.n_slots, p.n_eval, nsteps, ds | (narrow ? 4 : 0)) > TILE_SMEM_MAX)
                    continue;
                const uint64_t tiles = o.lanes / (32ull * tw);
                const uint64_t slots = (uint64_t)ng * (uint64_t)sms;
                const uint64_t waves = (tiles + slots - 1) / slots;
                const uint64_t per_wave = o.lanes / waves;
                // descriptor source weights (profiles/r02_kernelT_configs_C2.txt,
                // r02_mid_size_fresh_process.jsonl): resident >= a small table (<= 128 KB) read
                // through L1/L2 (C2, narrow descriptors, 2 groups: 3.86e13 vs 3.65e13; 5k gates,
                // 512-lane tiles: 6.31e12 vs 6.27e12) > TMA stream (3.21e13; 5.0e12) > a large
                // table from L2 (10k gates: TMA 7.1e12 vs global 6.3e12)
                const bool small_table = table_bytes <= 131072;
                const uint64_t wgt = ds == 1 ? 40 : ds == 0 ? (small_table ? 38 : 28) : 32;
                const uint64_t pref = ds == 1 ? 3 : ds == 0 && small_table ? 2 : ds == 2 ? 1 : 0;
                // ties (e.g. every plan fits one wave): more SMs busy, then wider tiles (C1,
                // 1,024 lanes: 8 tiles of 128 lanes 1.03e10 vs one 1,024-lane tile 7.8e9)
                const uint64_t busy = std::min<uint64_t>((tiles + ng - 1) / ng, (uint64_t)sms);
                const uint64_t score = (((per_wave / 64) * wgt) << 28) | (busy << 16) | ((uint64_t)tw << 8) |
                                       (pref << 4) | (uint64_t)(8 - ng);
                if (score > best) { best = score; pl.tw = tw; pl.ng = ng; pl.desc_smem = ds; }
            }
        }
    }
    if (!best) return fail(GS_ERR_ARG, "TILE: live state of a 128-lane tile exceeds shared memory (or lanes % 128)");
    pl.steps = pl.desc_smem == 2 ? st_chunk : st_level;
    if (narrow) pl.desc_smem |= 4;
    return GS_OK;
}

// GS_KERNEL_AUTO: kernel T when one tile's live state fits shared memory next to either the
// whole descriptor table or the TMA descriptor double buffer and the levels are narrow
// (small and mid-size circuits: measured 1.8x kernel A on C2, 5.8x on C1, 2.7x / 1.8x on
// 5k / 10k-gate synthetic circuits), else kernel A (large circuits are HBM-bound and T
// cannot hold them; from ~500 gates per level kernel A with concurrent lane groups wins:
// 20k gates / 38 levels at 65,536 lanes A 9.4e12 vs T 8.6e12, profiles/r01_mid_size_*).
// Programs with 6-8-input LUTs use kernel A.
gs_sim_opts resolve_auto(const Program& p, const gs_sim_opts& o) {
    gs_sim_opts r = o;
    if (o.kernel != GS_KERNEL_AUTO) return r;
    r.kernel = GS_KERNEL_LUT;
    // wide LUTs make every level ALU-heavy (2^k - 1 LOP3 per 32 lanes): kernel A's higher
    // occupancy wins from k = 6 on (measured on C2 collapsed to L = 6, 7, 8)
    if (p.max_k > 5) return r;
    uint32_t nl = 0;
    for (uint32_t l = 0; l < p.n_levels; ++l) nl += p.level_off[l + 1] > p.level_off[l] ? 1 : 0;
    if (nl && p.n_eval / nl > 400 && o.lanes >= 32768) return r;
    r.kernel = GS_KERNEL_TILE;
    Plans pl;
    const std::string saved = gs_last_error();
    // (a large descriptor table read from global memory is slow: T only with resident or
    // TMA-streamed descriptors, or a table small enough to stay cache-resident)
    if (p.n_eval == 0 || make_plans(p, r, pl) != GS_OK ||
        ((pl.desc_smem & 3) == 0 && (uint64_t)p.n_eval * ((pl.desc_smem & 4) ? 8 : 16) > 131072))
        r.kernel = GS_KERNEL_LUT;
    set_error(saved);
    return r;
}

Layout make_layout(const Program& p, const gs_sim_opts& o, const Plans& pl) {
    const TilePlan& t = pl.tile;
    Layout L{};
    const uint64_t words = o.lanes / 64;
    const uint64_t stride = words * 8;
    const bool poly = o.kernel == GS_KERNEL_POLY || o.kernel == GS_KERNEL_AB;
    size_t off = 0;
    auto take = [&](size_t bytes) {
        size_t at = off;
        off = align256(off + bytes);
        return at;
    };
    L.ctl = take(sizeof(Ctl));
    L.state = take((size_t)p.n_rows * stride);
    L.din = take((size_t)p.n_eval * 16);
    L.aux = take((size_t)p.n_eval * 16);
    L.dhi = take(p.any_wide ? (size_t)p.n_eval * 16 : 0);
    L.dtt = take(p.max_k > GS_MAX_K_LUT64 ? (size_t)p.n_eval * 32 : 0);
    L.term_off = take(poly ? ((size_t)p.n_eval + 1) * 4 : 0);
    L.terms = take(poly ? p.terms.size() * 4 : 0);
    L.po_rows = take((size_t)p.n_po * 4);
    L.latch_src = take(p.latch_src.size() * 4);
    L.latch_dst = take(p.latch_dst.size() * 4);
    L.reg_init = take(p.reg_init.size());
    L.trace_slot = take((size_t)words * 4);
    L.misr = take((size_t)2 * 64 * words * 8);        // double-buffered by cycle parity
    L.trace = take((size_t)o.trace_cycles * p.n_po * o.n_trace_words * 8);
    L.lane_sigs = take((size_t)o.lanes * 8);
    L.scratch = take((size_t)p.n_po * words * 8);
    L.t_desc = take(t.desc_n.empty() ? t.desc.size() * sizeof(TileDesc) : t.desc_n.size() * 4);
    L.t_desc_hi = take(t.desc_hi.size() * 4);   // 48 B per gate when any k > 4
    L.t_po = take(t.po_slot.size() * 4);
    L.t_lsrc = take(t.latch_src.size() * 4);
    L.t_ldst = take(t.latch_dst.size() * 4);
    L.t_wbrow = take(t.wb_row.size() * 4);
    L.t_wbslot = take(t.wb_slot.size() * 4);
    L.t_steps = take(pl.steps.size() * sizeof(uint2));
    L.total = off;
    return L;
}

}  // namespace

struct gs_sim {
    const Program* prog = nullptr;
    gs_sim_opts opts{};
    std::vector<uint32_t> trace_words;
    Layout L{};
    uint8_t* ws = nullptr;
    cudaStream_t stream = nullptr, cap = nullptr;
    uint32_t words = 0;
    uint64_t stride = 0;
    uint64_t cycle = 0;               // host mirror of Ctl::cycle
    int bound = 0;                    // 0 none, 1 generated, 2 host/device buffer
    uint64_t bound_seed = 0, bound_ptr = 0, bound_base = 0, bound_cycles = 0;
    uint64_t bind_stage[3] = {0, 0, 0};
    uint32_t bind_mode = 0;
    void* host_stage = nullptr;       // library-owned device copy of host stimulus
    size_t host_stage_bytes = 0;
    // gs_sim_run_streamed: library-owned double-buffered device staging + a copy stream
    void* stream_buf = nullptr;
    size_t stream_buf_bytes = 0;
    cudaStream_t copy = nullptr;
    cudaEvent_t ev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
    cudaGraphExec_t exec[2] = {nullptr, nullptr};
    TilePlan tile;
    uint32_t tw = 0, tile_grid = 0;
    int desc_smem = 0;
    uint32_t tile_groups = 1;
    std::vector<uint2> tile_steps;    // kernel T: level steps (uploaded to L.t_steps)
    uint32_t pdl = 1;                 // programmatic dependent launch between cycle kernels
    uint32_t min_warps = 0;           // kernel A auto-U threshold (2 waves of resident warps)
    uint32_t resident_blocks = 0;     // kernel A wide path: CTAs resident on the GPU
    uint32_t sms = 148;
    uint32_t groups = 1;              // concurrent lane groups (kernel A), one graph branch each
    std::vector<cudaStream_t> gstream;  // [groups - 1] branch streams (group 0: the caller's)
    std::vector<cudaEvent_t> gev;       // [0] fork, [1 .. groups - 1] joins
    uint64_t grid_stride_launches = 0;  // level launches whose grid was capped at residency
    uint64_t multi_gate_launches = 0;   // level launches with several gates per warp unit
    uint32_t cluster_size = 0, clusters = 0, slab_vec = 0, n_slabs = 0;   // kernel C
    // kernel A segmented slab schedule: slabs of lut_slab_vec 16-byte vectors (lut_slabs per
    // lane group); levels with slabbed[l] != 0 run slab-major in runs of consecutive such levels
    uint32_t lut_slabs = 1, lut_slab_vec = 0;
    std::vector<uint8_t> slabbed;

    Ctl* ctl() const { return reinterpret_cast<Ctl*>(ws + L.ctl); }
    uint8_t* state() const { return ws + L.state; }
    template <class T> T* at(size_t off) const { return reinterpret_cast<T*>(ws + off); }
};

#define CU(call)                                                                           \
    do {                                                                                   \
        cudaError_t e_ = (call);                                                           \
        if (e_ != cudaSuccess)                                                             \
            return fail(GS_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_));  \
    } while (0)

static LevelArgs level_args(const gs_sim* s, uint32_t l, uint32_t parity) {
    const Program& p = *s->prog;
    LevelArgs a{};
    a.din = s->at<const uint4>(s->L.din);
    a.aux = s->at<const GateAux>(s->L.aux);
    a.dhi = p.any_wide ? s->at<const uint4>(s->L.dhi) : nullptr;
    a.dtt = p.max_k > GS_MAX_K_LUT64 ? s->at<const uint4>(s->L.dtt) : nullptr;
    a.term_off = s->at<const uint32_t>(s->L.term_off);
    a.terms = s->at<const uint32_t>(s->L.terms);
    a.g0 = p.level_off[l];
    a.ng = p.level_off[l + 1] - p.level_off[l];
    a.state = s->state();
    a.stride = s->stride;
    a.words = s->words;
    a.row_gate0 = p.row_gate0;
    a.qcur = parity ? p.n_reg : 0;
    a.qnext = parity ? 0 : p.n_reg;
    a.ctl = s->ctl();
    a.pdl = s->pdl;
    a.min_warps = s->min_warps;
    a.grid_blocks = (s->opts.flags & GS_SIM_NO_GRID_STRIDE) ? 0u : s->resident_blocks;
    a.sms = s->sms;
    return a;
}

static EndArgs end_args(const gs_sim* s, uint32_t parity) {
    const Program& p = *s->prog;
    EndArgs e{};
    e.ctl = s->ctl();
    e.state = s->state();
    e.stride = s->stride;
    e.words = s->words;
    e.latch_src = s->at<const uint32_t>(s->L.latch_src);
    e.latch_dst = s->at<const uint32_t>(s->L.latch_dst);
    e.n_latch = (uint32_t)p.latch_src.size();
    e.row_q0 = p.row_q0;
    e.qcur = parity ? p.n_reg : 0;
    e.qnext = parity ? 0 : p.n_reg;
    e.po_rows = s->at<const uint32_t>(s->L.po_rows);
    e.n_po = p.n_po;
    e.misr_cur = s->at<unsigned long long>(s->L.misr) + (size_t)parity * 64 * s->words;
    e.misr_next = s->at<unsigned long long>(s->L.misr) + (size_t)(parity ^ 1) * 64 * s->words;
    e.trace_slot = s->at<const int32_t>(s->L.trace_slot);
    e.trace = (s->opts.n_trace_words && s->opts.trace_cycles) ? s->at<unsigned long long>(s->L.trace) : nullptr;
    e.ntw = s->opts.n_trace_words;
    e.trace_cap = s->opts.trace_cycles;
    e.pdl = s->pdl;
    return e;
}

// vec0 / vslab: the lane range of the launch in 16-byte vectors (vslab 0 = the whole row)
static cudaError_t level_launch(gs_sim* s, uint32_t l, uint32_t parity, cudaStream_t st, uint32_t vec0 = 0,
                                uint32_t vslab = 0) {
    LevelArgs a = level_args(s, l, parity);
    a.unroll = s->opts.lut_unroll;
    a.vec0 = vec0;
    a.vslab = vslab;
    uint32_t gs_flag = 0;
    cudaError_t e = cudaSuccess;
    switch (s->opts.kernel) {
        case GS_KERNEL_POLY: return launch_level_poly(a, 0, st);
        case GS_KERNEL_AB:
            e = launch_level_lut(a, st, &gs_flag);
            if (e != cudaSuccess) return e;
            e = launch_level_poly(a, 1, st);
            break;
        default: e = launch_level_lut(a, st, &gs_flag); break;
    }
    s->grid_stride_launches += gs_flag & 1u;
    s->multi_gate_launches += (gs_flag >> 1) & 1u;
    return e;
}

static cudaError_t tile_launch(const gs_sim* s, uint32_t ncycles, cudaStream_t st) {
    const Program& p = *s->prog;
    const TilePlan& t = s->tile;
    TileArgs a{};
    a.desc = s->at<const TileDesc>(s->L.t_desc);
    a.desc_hi = s->at<const uint4>(s->L.t_desc_hi);
    a.steps = s->at<const uint2>(s->L.t_steps);
    a.n_eval = p.n_eval;
    a.n_steps = (uint32_t)s->tile_steps.size();
    a.desc_smem = (uint32_t)s->desc_smem;
    a.po_slot = s->at<const uint32_t>(s->L.t_po);
    a.n_po = p.n_po;
    a.latch_src = s->at<const uint32_t>(s->L.t_lsrc);
    a.latch_dst = s->at<const uint32_t>(s->L.t_ldst);
    a.n_latch = (uint32_t)t.latch_src.size();
    a.wb_row = s->at<const uint32_t>(s->L.t_wbrow);
    a.wb_slot = s->at<const uint32_t>(s->L.t_wbslot);
    a.n_wb = (uint32_t)t.wb_row.size();
    a.n_pi = p.n_pi;
    a.n_reg = p.n_reg;
    a.q0 = t.q0;
    a.n_slots = t.n_slots;
    a.state = s->state();
    a.words = s->words;
    a.row_q0 = p.row_q0;
    a.ctl = s->ctl();
    a.tile_next = &s->ctl()->tile_next;
    a.misr = s->at<unsigned long long>(s->L.misr);
    a.trace_slot = s->at<const int32_t>(s->L.trace_slot);
    a.trace = (s->opts.n_trace_words && s->opts.trace_cycles) ? s->at<unsigned long long>(s->L.trace) : nullptr;
    a.ntw = s->opts.n_trace_words;
    a.trace_cap = s->opts.trace_cycles;
    a.word_off = s->opts.lane_offset / 64;
    a.ncycles = ncycles;
    a.n_tiles = (uint32_t)(s->opts.lanes / (32ull * s->tw));
    return launch_tile(a, s->tw, s->tile_groups, s->tile_grid, st);
}

static cudaError_t cluster_launch(const gs_sim* s, uint32_t ncycles, cudaStream_t st) {
    const Program& p = *s->prog;
    ClusterArgs a{};
    a.din = s->at<const uint4>(s->L.din);
    a.aux = s->at<const GateAux>(s->L.aux);
    a.dhi = p.any_wide ? s->at<const uint4>(s->L.dhi) : nullptr;
    a.dtt = p.max_k > GS_MAX_K_LUT64 ? s->at<const uint4>(s->L.dtt) : nullptr;
    a.steps = s->at<const uint2>(s->L.t_steps);
    a.n_steps = (uint32_t)s->tile_steps.size();
    a.state = s->state();
    a.stride = s->stride;
    a.words = s->words;
    a.row_gate0 = p.row_gate0;
    a.row_pi0 = p.row_pi0;
    a.n_pi = p.n_pi;
    a.row_q0 = p.row_q0;
    a.n_reg = p.n_reg;
    a.latch_src = s->at<const uint32_t>(s->L.latch_src);
    a.latch_dst = s->at<const uint32_t>(s->L.latch_dst);
    a.n_latch = (uint32_t)p.latch_src.size();
    a.po_rows = s->at<const uint32_t>(s->L.po_rows);
    a.n_po = p.n_po;
    a.misr = s->at<unsigned long long>(s->L.misr);
    a.trace_slot = s->at<const int32_t>(s->L.trace_slot);
    a.trace = (s->opts.n_trace_words && s->opts.trace_cycles) ? s->at<unsigned long long>(s->L.trace) : nullptr;
    a.ntw = s->opts.n_trace_words;
    a.trace_cap = s->opts.trace_cycles;
    a.ctl = s->ctl();
    a.tile_next = &s->ctl()->tile_next;
    a.word_off = s->opts.lane_offset / 64;
    a.ncycles = ncycles;
    a.slab_vec = s->slab_vec;
    a.n_slabs = s->n_slabs;
    return launch_cluster(a, s->clusters, s->cluster_size, st);
}

// The level chain of one cycle over the lane range [v0, v0 + vlen) (16-byte vectors; vlen 0
// = the whole row).  With the segmented slab schedule a run of consecutive wide levels goes
// slab after slab (each slab through every level of the run) and the other levels over the
// whole range; levels only read earlier levels of the same lanes, so any slab order is valid.
static cudaError_t level_chain(gs_sim* s, uint32_t parity, cudaStream_t st, uint32_t v0, uint32_t vlen) {
    const Program& p = *s->prog;
    const uint32_t nslab = s->lut_slab_vec ? (vlen ? vlen : s->words / 2) / s->lut_slab_vec : 1;
    cudaError_t e = cudaSuccess;
    for (uint32_t l = 0; l < p.n_levels;) {
        if (nslab <= 1 || !s->slabbed[l]) {
            if ((e = level_launch(s, l, parity, st, v0, vlen)) != cudaSuccess) return e;
            ++l;
            continue;
        }
        uint32_t m = l;
        while (m < p.n_levels && s->slabbed[m]) ++m;
        for (uint32_t j = 0; j < nslab; ++j)
            for (uint32_t ll = l; ll < m; ++ll)
                if ((e = level_launch(s, ll, parity, st, v0 + j * s->lut_slab_vec, s->lut_slab_vec)) != cudaSuccess)
                    return e;
        l = m;
    }
    return e;
}

// evs (profiling): timing events around every level launch (one group), or around the
// concurrent level region (lane groups); ext = the launches are being captured, record the
// events as graph nodes
static cudaError_t cycle_launches(gs_sim* s, uint32_t parity, cudaStream_t st,
                                  std::vector<cudaEvent_t>* evs = nullptr, bool ext = false) {
    const Program& p = *s->prog;
    cudaError_t e = launch_stim(s->ctl(), s->state(), s->stride, s->words, p.row_pi0, p.n_pi,
                                s->opts.lane_offset / 64, s->pdl, st);
    if (e != cudaSuccess) return e;
    if (s->groups > 1) {
        // lane groups: one branch per group, forked after the stimulus kernel and joined
        // before the end-of-cycle kernel; the branches share nothing but the stimulus rows
        if (evs) cudaEventRecordWithFlags((*evs)[0], st, ext ? cudaEventRecordExternal : 0u);
        if ((e = cudaEventRecord(s->gev[0], st)) != cudaSuccess) return e;
        const uint32_t vs = (s->words / 2) / s->groups;
        for (uint32_t br = 0; br < s->groups; ++br) {
            cudaStream_t b = br ? s->gstream[br - 1] : st;
            if (br && (e = cudaStreamWaitEvent(b, s->gev[0], 0)) != cudaSuccess) return e;
            if ((e = level_chain(s, parity, b, br * vs, vs)) != cudaSuccess) return e;
            if (br && (e = cudaEventRecord(s->gev[br], b)) != cudaSuccess) return e;
        }
        for (uint32_t br = 1; br < s->groups; ++br)
            if ((e = cudaStreamWaitEvent(st, s->gev[br], 0)) != cudaSuccess) return e;
        if (evs) cudaEventRecordWithFlags((*evs)[1], st, ext ? cudaEventRecordExternal : 0u);
        return launch_end_cycle(end_args(s, parity), st);
    }
    if (s->lut_slabs > 1) {
        if (evs) cudaEventRecordWithFlags((*evs)[0], st, ext ? cudaEventRecordExternal : 0u);
        if ((e = level_chain(s, parity, st, 0, 0)) != cudaSuccess) return e;
        if (evs) cudaEventRecordWithFlags((*evs)[1], st, ext ? cudaEventRecordExternal : 0u);
        return launch_end_cycle(end_args(s, parity), st);
    }
    for (uint32_t l = 0; l < p.n_levels; ++l) {
        if (evs) cudaEventRecord((*evs)[2 * (size_t)l], st);
        e = level_launch(s, l, parity, st);
        if (e != cudaSuccess) return e;
        if (evs) cudaEventRecord((*evs)[2 * (size_t)l + 1], st);
    }
    return launch_end_cycle(end_args(s, parity), st);
}

static gs_status ensure_graph(gs_sim* s, uint32_t parity) {
    if (s->exec[parity]) return GS_OK;
    cudaGraph_t g = nullptr;
    CU(cudaStreamBeginCapture(s->cap, cudaStreamCaptureModeThreadLocal));
    cudaError_t e = cycle_launches(s, parity, s->cap);
    cudaError_t e2 = cudaStreamEndCapture(s->cap, &g);
    if (e != cudaSuccess) {
        if (g) cudaGraphDestroy(g);
        return fail(GS_ERR_CUDA, std::string("graph capture: ") + cudaGetErrorString(e));
    }
    CU(e2);
    cudaError_t e3 = cudaGraphInstantiate(&s->exec[parity], g, 0);
    cudaGraphDestroy(g);
    CU(e3);
    return GS_OK;
}

// lane_groups = 0: concurrent lane groups for kernel A (measured on C2-C5):
// four groups of >= 4,096 lanes, but only two when a level launch averages > 1 GB of
// algorithmic traffic (C5 shard: the level already fills the GPU for ~0.3 ms, and four
// groups' 1 KB row segments lose more to short rows than the overlap gains).
static uint32_t auto_lane_groups(const Program& p, const gs_sim_opts& o) {
    if (o.kernel != GS_KERNEL_LUT || o.lanes % 128) return 1;
    const uint32_t vrow = (uint32_t)(o.lanes / 128);
    double bytes = 0;
    uint32_t nl = 0;
    for (uint32_t l = 0; l < p.n_levels; ++l) nl += p.level_off[l + 1] > p.level_off[l] ? 1 : 0;
    for (uint32_t g = 0; g < p.n_eval; ++g) bytes += (double)((p.aux[g].k & 0xFFu) + 1) * (double)(o.lanes / 8);
    const uint32_t gmax = (nl && bytes / nl > 1e9) ? 2 : 4;
    for (uint32_t G = gmax; G > 1; G /= 2)
        if (vrow % G == 0 && (vrow / G) % 32 == 0) return G;
    return 1;
}

static void destroy_groups(gs_sim* s) {
    for (auto& b : s->gstream)
        if (b) cudaStreamSynchronize(b), cudaStreamDestroy(b);
    for (auto& v : s->gev)
        if (v) cudaEventDestroy(v);
    s->gstream.clear();
    s->gev.clear();
}

static void free_sim(gs_sim* s) {
    if (!s) return;
    destroy_groups(s);
    for (auto& x : s->exec)
        if (x) cudaGraphExecDestroy(x);
    if (s->cap) cudaStreamDestroy(s->cap);
    if (s->host_stage) cudaFree(s->host_stage);
    if (s->copy) cudaStreamSynchronize(s->copy);
    if (s->stream_buf) cudaFree(s->stream_buf);
    for (auto& e : s->ev)
        if (e) cudaEventDestroy(e);
    if (s->copy) cudaStreamDestroy(s->copy);
    delete s;
}

static gs_status check_sim(const gs_sim* s, const char* fn) {
    if (!s) return fail(GS_ERR_ARG, std::string(fn) + ": NULL sim");
    return GS_OK;
}

// Ctl fields seed, stim_ptr, stim_base are contiguous, stim_mode follows later
static gs_status write_binding(gs_sim* s) {
    static_assert(offsetof(Ctl, stim_ptr) == offsetof(Ctl, seed) + 8, "Ctl layout");
    static_assert(offsetof(Ctl, stim_base) == offsetof(Ctl, seed) + 16, "Ctl layout");
    s->bind_stage[0] = s->bound_seed;
    s->bind_stage[1] = s->bound_ptr;
    s->bind_stage[2] = s->bound_base;
    s->bind_mode = s->bound == 2 ? 1u : 0u;
    CU(cudaMemcpyAsync(s->ws + s->L.ctl + offsetof(Ctl, seed), s->bind_stage, 24, cudaMemcpyHostToDevice, s->stream));
    CU(cudaMemcpyAsync(s->ws + s->L.ctl + offsetof(Ctl, stim_mode), &s->bind_mode, 4, cudaMemcpyHostToDevice, s->stream));
    CU(cudaStreamSynchronize(s->stream));   // the staging fields may be rewritten by the next bind
    return GS_OK;
}

// flag bits of gs_sim_opts retired in 0.2.0 (L2 hints, bulk-copy gathers, global T slots)
constexpr uint32_t GS_SIM_RETIRED_FLAGS = 2u | 4u | 64u | 128u | 256u;
constexpr uint32_t GS_SIM_KNOWN_FLAGS = GS_SIM_NO_PDL | GS_SIM_NO_GRID_STRIDE | GS_SIM_TILE_DESC_GLOBAL |
                                        GS_SIM_TILE_DESC_TMA | GS_SIM_TILE_DESC_RESIDENT;

static gs_status check_opts(const gs_sim_opts* o, const char* fn) {
    if (o->lanes == 0 || o->lanes % 64) return fail(GS_ERR_ARG, std::string(fn) + ": lanes must be a positive multiple of 64");
    if (o->lanes / 64 >= (1ull << 31)) return fail(GS_ERR_ARG, std::string(fn) + ": too many lanes");
    if (o->lane_offset % 64) return fail(GS_ERR_ARG, std::string(fn) + ": lane_offset must be a multiple of 64");
    if (o->kernel < GS_KERNEL_AUTO || o->kernel > GS_KERNEL_CLUSTER || o->kernel == 4)
        return fail(GS_ERR_ARG, std::string(fn) + ": bad kernel");
    if (o->flags & GS_SIM_RETIRED_FLAGS)
        return fail(GS_ERR_ARG, std::string(fn) + ": flag retired in 0.2.0 (L2 hints / bulk gathers / global T slots)");
    if (o->flags & ~GS_SIM_KNOWN_FLAGS) return fail(GS_ERR_ARG, std::string(fn) + ": unknown flag");
    if (o->n_trace_words && !o->trace_words) return fail(GS_ERR_ARG, std::string(fn) + ": trace_words is NULL");
    return GS_OK;
}

// ======================================================================= ABI bodies
// (each wrapped in GS_TRY by its extern "C" entry point below)

static gs_status sim_workspace_bytes(const gs_program* prog, const gs_sim_opts* opts, size_t* bytes) {
    if (!prog || !opts || !bytes) return fail(GS_ERR_ARG, "gs_sim_workspace_bytes: NULL argument");
    if (gs_status st = check_opts(opts, "gs_sim_workspace_bytes")) return st;
    const gs_sim_opts o = resolve_auto(*prog->p, *opts);
    Plans pl;
    if (gs_status st = make_plans(*prog->p, o, pl)) return st;
    *bytes = make_layout(*prog->p, o, pl).total;
    clear_error();
    return GS_OK;
}

static gs_status sim_reset(gs_sim* s);

static gs_status sim_create(const gs_program* prog, const gs_sim_opts* opts_in, void* dev_ws, size_t bytes, gs_sim** out) {
    NvtxRange nvtx("gs_sim_create");
    if (!prog || !opts_in || !out || !dev_ws) return fail(GS_ERR_ARG, "gs_sim_create: NULL argument");
    if (gs_status st = check_opts(opts_in, "gs_sim_create")) return st;
    const gs_sim_opts resolved = resolve_auto(*prog->p, *opts_in);
    const gs_sim_opts* opts = &resolved;
    if ((reinterpret_cast<uintptr_t>(dev_ws) & 255) != 0) return fail(GS_ERR_ARG, "gs_sim_create: workspace must be 256-byte aligned");
    const Program& p = *prog->p;
    const uint32_t words = (uint32_t)(opts->lanes / 64);
    for (uint32_t i = 0; i < opts->n_trace_words; ++i)
        if (opts->trace_words[i] >= words) return fail(GS_ERR_ARG, "gs_sim_create: trace word out of range");
    Plans pls;
    if (gs_status st = make_plans(p, *opts, pls)) return st;
    Layout L = make_layout(p, *opts, pls);
    if (bytes < L.total) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_sim_create: workspace smaller than gs_sim_workspace_bytes");
    const bool lut_slab = opts->kernel == GS_KERNEL_LUT && opts->slab_lanes;
    uint32_t groups = opts->lane_groups;
    if (groups == 0) groups = lut_slab ? 1 : auto_lane_groups(p, *opts);
    if (lut_slab && (opts->slab_lanes % 4096 || (opts->lanes / groups) % opts->slab_lanes || opts->lanes % groups))
        return fail(GS_ERR_ARG, "gs_sim_create: LUT slab_lanes must be a multiple of 4096 dividing the lanes "
                                "of a lane group");
    if (groups > 1) {
        const uint32_t vrow = words / 2;
        if (opts->kernel != GS_KERNEL_LUT || words % 2 || vrow % groups || (vrow / groups) % 32)
            return fail(GS_ERR_ARG, "gs_sim_create: lane_groups needs kernel A, (lanes/128) % groups == 0 "
                                    "and a multiple of 4096 lanes per group");
    }
    CU(cudaSetDevice(opts->device));
    gs_sim* s = new gs_sim();
    struct Guard {                        // frees the half-built sim on every early return
        gs_sim*& s;
        ~Guard() { free_sim(s); }
    } guard{s};
    s->prog = &p;
    s->opts = *opts;
    s->trace_words.assign(opts->trace_words, opts->trace_words + opts->n_trace_words);
    s->opts.trace_words = s->trace_words.data();
    s->L = L;
    s->ws = static_cast<uint8_t*>(dev_ws);
    s->stream = static_cast<cudaStream_t>(opts->stream);
    s->words = words;
    s->stride = (uint64_t)words * 8;
    s->tile = pls.tile;
    s->tw = pls.tw;
    s->desc_smem = pls.desc_smem;
    s->tile_steps = pls.steps;
    s->pdl = (opts->flags & GS_SIM_NO_PDL) ? 0u : 1u;
    s->groups = groups;
    if (lut_slab && opts->slab_lanes < opts->lanes / groups) {
        s->lut_slabs = (uint32_t)(opts->lanes / groups / opts->slab_lanes);
        s->lut_slab_vec = opts->slab_lanes / 128;
        const uint32_t wmin = opts->slab_min_gates ? opts->slab_min_gates : 32768u;
        s->slabbed.assign(p.n_levels, 0);
        for (uint32_t l = 0; l < p.n_levels; ++l) s->slabbed[l] = p.level_off[l + 1] - p.level_off[l] >= wmin;
    }
    {
        int sms = 148;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, opts->device);
        s->min_warps = (uint32_t)sms * 32u * 2u;   // 4 CTAs x 8 warps per SM, two waves
        s->resident_blocks = level_lut_resident_blocks(opts->device);
        s->sms = (uint32_t)sms;
    }
    cudaError_t e = cudaSuccess;
    if (s->opts.kernel == GS_KERNEL_TILE) {
        uint32_t per = 0;
        s->tile_groups = pls.ng;
        e = tile_setup(s->tw, s->tile_groups, s->tile.n_slots, p.n_eval, (uint32_t)s->tile_steps.size(),
                       s->desc_smem, p.n_reg > 0, &per);
        if (e != cudaSuccess || per == 0)
            return fail(e != cudaSuccess ? GS_ERR_CUDA : GS_ERR_ARG,
                        std::string("TILE: kernel setup: ") + (e != cudaSuccess ? cudaGetErrorString(e) : "0 CTAs fit an SM"));
        const uint32_t tiles = (uint32_t)(opts->lanes / (32ull * s->tw));
        s->tile_grid = std::min<uint32_t>((tiles + s->tile_groups - 1) / s->tile_groups, per * s->sms);
    }
    if (s->opts.kernel == GS_KERNEL_CLUSTER) {
        const uint64_t sl = opts->slab_lanes ? opts->slab_lanes : 256;
        s->cluster_size = opts->cluster_size ? opts->cluster_size : 2;
        s->slab_vec = (uint32_t)(sl / 128);
        s->n_slabs = (uint32_t)(opts->lanes / sl);
        uint32_t maxc = 0;
        e = cluster_max_active(s->slab_vec, s->cluster_size, &maxc);
        if (e != cudaSuccess || maxc == 0)
            return fail(e != cudaSuccess ? GS_ERR_CUDA : GS_ERR_ARG,
                        std::string("CLUSTER: no cluster fits: ") + (e != cudaSuccess ? cudaGetErrorString(e) : "0 active"));
        s->clusters = std::min(maxc, s->n_slabs);
        s->tile_steps = pls.steps;
    }
    CU(cudaStreamCreateWithFlags(&s->cap, cudaStreamNonBlocking));
    if (s->groups > 1) {
        s->gstream.assign(s->groups - 1, nullptr);
        s->gev.assign(s->groups, nullptr);
        for (auto& b : s->gstream) CU(cudaStreamCreateWithFlags(&b, cudaStreamNonBlocking));
        for (auto& v : s->gev) CU(cudaEventCreateWithFlags(&v, cudaEventDisableTiming));
    }
    // upload the program (descriptors are device-resident for the sim's lifetime)
    struct Up { size_t off; const void* src; size_t n; };
    std::vector<int32_t> slot(words, -1);
    for (uint32_t i = 0; i < opts->n_trace_words; ++i) slot[opts->trace_words[i]] = (int32_t)i;
    const bool poly = s->opts.kernel == GS_KERNEL_POLY || s->opts.kernel == GS_KERNEL_AB;
    std::vector<Up> ups = {
        {L.din, p.in_lo.data(), p.in_lo.size() * 4},
        {L.aux, p.aux.data(), p.aux.size() * sizeof(GateAux)},
        {L.dhi, p.in_hi.data(), p.any_wide ? p.in_hi.size() * 4 : 0},
        {L.dtt, p.tt_full.data(), p.max_k > GS_MAX_K_LUT64 ? p.tt_full.size() * 8 : 0},
        {L.term_off, p.term_off.data(), poly ? p.term_off.size() * 4 : 0},
        {L.terms, p.terms.data(), poly ? p.terms.size() * 4 : 0},
        {L.po_rows, p.po_rows.data(), p.po_rows.size() * 4},
        {L.latch_src, p.latch_src.data(), p.latch_src.size() * 4},
        {L.latch_dst, p.latch_dst.data(), p.latch_dst.size() * 4},
        {L.reg_init, p.reg_init.data(), p.reg_init.size()},
        {L.trace_slot, slot.data(), slot.size() * 4},
        {L.t_desc, s->tile.desc_n.empty() ? (const void*)s->tile.desc.data() : (const void*)s->tile.desc_n.data(),
         s->tile.desc_n.empty() ? s->tile.desc.size() * sizeof(TileDesc) : s->tile.desc_n.size() * 4},
        {L.t_desc_hi, s->tile.desc_hi.data(), s->tile.desc_hi.size() * 4},
        {L.t_po, s->tile.po_slot.data(), s->tile.po_slot.size() * 4},
        {L.t_lsrc, s->tile.latch_src.data(), s->tile.latch_src.size() * 4},
        {L.t_ldst, s->tile.latch_dst.data(), s->tile.latch_dst.size() * 4},
        {L.t_wbrow, s->tile.wb_row.data(), s->tile.wb_row.size() * 4},
        {L.t_wbslot, s->tile.wb_slot.data(), s->tile.wb_slot.size() * 4},
        {L.t_steps, s->tile_steps.data(), s->tile_steps.size() * sizeof(uint2)},
    };
    for (const Up& u : ups)
        if (u.n) CU(cudaMemcpyAsync(s->ws + u.off, u.src, u.n, cudaMemcpyHostToDevice, s->stream));
    CU(cudaStreamSynchronize(s->stream));   // host vectors above are temporaries
    if (gs_status st = sim_reset(s)) return st;
    *out = s;
    s = nullptr;                            // ownership passes to the caller
    clear_error();
    return GS_OK;
}

static gs_status sim_reset(gs_sim* s) {
    if (gs_status st = check_sim(s, "gs_sim_reset")) return st;
    const Program& p = *s->prog;
    CU(cudaSetDevice(s->opts.device));
    CU(cudaMemsetAsync(s->ws + s->L.ctl, 0, sizeof(Ctl), s->stream));
    CU(cudaMemsetAsync(s->ws + s->L.misr, 0, (size_t)2 * 64 * s->words * 8, s->stream));
    CU(cudaMemsetAsync(s->ws + s->L.lane_sigs, 0, (size_t)s->opts.lanes * 8, s->stream));
    size_t tbytes = (size_t)s->opts.trace_cycles * p.n_po * s->opts.n_trace_words * 8;
    if (tbytes) CU(cudaMemsetAsync(s->ws + s->L.trace, 0, tbytes, s->stream));
    CU(launch_fill_rows(s->state(), s->stride, s->words, 0, 1, nullptr, 0, s->stream));          // const0
    CU(launch_fill_rows(s->state(), s->stride, s->words, 1, 1, nullptr, 1, s->stream));          // const1
    CU(launch_fill_rows(s->state(), s->stride, s->words, p.row_q0, p.n_reg, s->at<const uint8_t>(s->L.reg_init), 0, s->stream));
    s->cycle = 0;
    // keep the binding; a bound buffer restarts at its first cycle
    s->bound_base = 0;
    if (s->bound)
        if (gs_status st = write_binding(s)) return st;
    clear_error();
    return GS_OK;
}

static gs_status sim_set_lane_offset(gs_sim* s, uint64_t lane_offset) {
    if (gs_status st = check_sim(s, "gs_sim_set_lane_offset")) return st;
    if (lane_offset % 64) return fail(GS_ERR_ARG, "gs_sim_set_lane_offset: lane_offset must be a multiple of 64");
    CU(cudaSetDevice(s->opts.device));
    if (lane_offset != s->opts.lane_offset) {
        // the offset is a launch argument baked into the captured cycle graphs
        CU(cudaStreamSynchronize(s->stream));
        for (auto& x : s->exec)
            if (x) {
                cudaGraphExecDestroy(x);
                x = nullptr;
            }
        s->opts.lane_offset = lane_offset;
    }
    return sim_reset(s);
}

static gs_status sim_bind_generated(gs_sim* s, uint64_t seed) {
    if (gs_status st = check_sim(s, "gs_sim_bind_stimulus_generated")) return st;
    CU(cudaSetDevice(s->opts.device));
    s->bound = 1;
    s->bound_seed = seed;
    s->bound_ptr = 0;
    s->bound_base = s->cycle;
    s->bound_cycles = 0;
    if (gs_status st = write_binding(s)) return st;
    clear_error();
    return GS_OK;
}

static gs_status sim_bind_device(gs_sim* s, const uint64_t* dev_words, uint32_t cycles) {
    if (gs_status st = check_sim(s, "gs_sim_bind_stimulus_device")) return st;
    if (!dev_words && cycles) return fail(GS_ERR_ARG, "gs_sim_bind_stimulus_device: NULL words");
    CU(cudaSetDevice(s->opts.device));
    s->bound = 2;
    s->bound_seed = 0;
    s->bound_ptr = reinterpret_cast<uint64_t>(dev_words);
    s->bound_base = s->cycle;
    s->bound_cycles = cycles;
    if (gs_status st = write_binding(s)) return st;
    clear_error();
    return GS_OK;
}

static gs_status sim_bind_host(gs_sim* s, const uint64_t* words, uint32_t cycles) {
    if (gs_status st = check_sim(s, "gs_sim_bind_stimulus_host")) return st;
    if (!words && cycles) return fail(GS_ERR_ARG, "gs_sim_bind_stimulus_host: NULL words");
    CU(cudaSetDevice(s->opts.device));
    const size_t bytes = (size_t)cycles * s->prog->n_pi * s->words * 8;
    if (bytes > s->host_stage_bytes) {
        CU(cudaStreamSynchronize(s->stream));
        if (s->host_stage) cudaFree(s->host_stage);
        s->host_stage = nullptr;
        s->host_stage_bytes = 0;
        CU(cudaMalloc(&s->host_stage, bytes));
        s->host_stage_bytes = bytes;
    }
    if (bytes) CU(cudaMemcpyAsync(s->host_stage, words, bytes, cudaMemcpyHostToDevice, s->stream));
    s->bound = 2;
    s->bound_seed = 0;
    s->bound_ptr = reinterpret_cast<uint64_t>(s->host_stage);
    s->bound_base = s->cycle;
    s->bound_cycles = cycles;
    if (gs_status st = write_binding(s)) return st;
    clear_error();
    return GS_OK;
}

static gs_status sim_step(gs_sim* s, uint32_t n) {
    NvtxRange nvtx("gs_sim_step");
    if (gs_status st = check_sim(s, "gs_sim_step")) return st;
    if (!s->bound) return fail(GS_ERR_STATE, "gs_sim_step: no stimulus bound");
    if (s->bound == 2 && s->cycle + n > s->bound_base + s->bound_cycles)
        return fail(GS_ERR_STATE, "gs_sim_step: stepping past the bound stimulus cycles");
    CU(cudaSetDevice(s->opts.device));
    if (s->opts.kernel == GS_KERNEL_TILE || s->opts.kernel == GS_KERNEL_CLUSTER) {
        // every cycle of the step in one launch
        CU(s->opts.kernel == GS_KERNEL_TILE ? tile_launch(s, n, s->stream) : cluster_launch(s, n, s->stream));
        s->cycle += n;
        clear_error();
        return GS_OK;
    }
    for (uint32_t i = 0; i < n; ++i) {
        const uint32_t parity = (uint32_t)(s->cycle & 1);
        if (s->opts.use_graphs) {
            if (gs_status st = ensure_graph(s, parity)) return st;
            CU(cudaGraphLaunch(s->exec[parity], s->stream));
        } else {
            CU(cycle_launches(s, parity, s->stream));
        }
        s->cycle++;
    }
    clear_error();
    return GS_OK;
}

static gs_status sim_run_streamed(gs_sim* s, const uint64_t* host_stim, uint64_t* host_out, uint32_t ncycles,
                                  uint32_t chunk) {
    NvtxRange nvtx("gs_sim_run_streamed");
    if (gs_status st = check_sim(s, "gs_sim_run_streamed")) return st;
    if (!host_stim && ncycles) return fail(GS_ERR_ARG, "gs_sim_run_streamed: NULL host_stim");
    if (!ncycles) return GS_OK;
    const Program& p = *s->prog;
    if (!chunk) chunk = 25;
    chunk = std::min(chunk, ncycles);
    const size_t w = s->words;
    const size_t in_b = (size_t)chunk * p.n_pi * w * 8, out_b = host_out ? (size_t)chunk * p.n_po * w * 8 : 0;
    const size_t in_b2 = (in_b + 255) & ~(size_t)255, out_b2 = (out_b + 255) & ~(size_t)255;
    CU(cudaSetDevice(s->opts.device));
    if (2 * (in_b2 + out_b2) > s->stream_buf_bytes) {
        CU(cudaStreamSynchronize(s->stream));
        if (s->copy) CU(cudaStreamSynchronize(s->copy));
        if (s->stream_buf) cudaFree(s->stream_buf);
        s->stream_buf = nullptr;
        s->stream_buf_bytes = 0;
        CU(cudaMalloc(&s->stream_buf, 2 * (in_b2 + out_b2)));
        s->stream_buf_bytes = 2 * (in_b2 + out_b2);
    }
    if (!s->copy) {
        CU(cudaStreamCreateWithFlags(&s->copy, cudaStreamNonBlocking));
        for (auto& e : s->ev) CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    const int prev_bound = s->bound;
    const uint64_t prev_seed = s->bound_seed;
    uint8_t* buf = static_cast<uint8_t*>(s->stream_buf);
    auto in_slot = [&](uint32_t i) { return buf + (i & 1) * in_b2; };
    auto out_slot = [&](uint32_t i) { return buf + 2 * in_b2 + (i & 1) * out_b2; };
    cudaEvent_t* ev_in = s->ev;          // H2D of the slot's stimuli done
    cudaEvent_t* ev_comp = s->ev + 2;    // compute that read / wrote the slot done
    cudaEvent_t* ev_out = s->ev + 4;     // D2H of the slot's outputs done
    const uint32_t nch = (ncycles + chunk - 1) / chunk;
    const uint64_t c_start = s->cycle;
    // the copy stream may not start before everything already queued on the sim's stream
    CU(cudaEventRecord(ev_comp[0], s->stream));
    CU(cudaEventRecord(ev_comp[1], s->stream));
    CU(cudaEventRecord(ev_out[0], s->stream));
    CU(cudaEventRecord(ev_out[1], s->stream));
    auto h2d = [&](uint32_t i) -> gs_status {
        const uint32_t cc = std::min<uint32_t>(chunk, ncycles - i * chunk);
        CU(cudaStreamWaitEvent(s->copy, ev_comp[i & 1], 0));          // slot no longer read
        CU(cudaMemcpyAsync(in_slot(i), host_stim + (size_t)i * chunk * p.n_pi * w, (size_t)cc * p.n_pi * w * 8,
                           cudaMemcpyHostToDevice, s->copy));
        CU(cudaEventRecord(ev_in[i & 1], s->copy));
        return GS_OK;
    };
    if (gs_status st = h2d(0)) return st;
    for (uint32_t i = 0; i < nch; ++i) {
        const uint32_t cc = std::min<uint32_t>(chunk, ncycles - i * chunk);
        const uint64_t c0 = c_start + (uint64_t)i * chunk;
        if (i + 1 < nch)
            if (gs_status st = h2d(i + 1)) return st;                  // overlaps chunk i's compute
        CU(cudaStreamWaitEvent(s->stream, ev_in[i & 1], 0));
        CU(cudaStreamWaitEvent(s->stream, ev_out[i & 1], 0));          // output slot drained
        CU(launch_set_binding(s->ctl(), reinterpret_cast<uint64_t>(in_slot(i)), c0, 1u,
                              host_out ? reinterpret_cast<uint64_t>(out_slot(i)) : 0ull, c0, cc, s->stream));
        s->bound = 2;
        s->bound_ptr = reinterpret_cast<uint64_t>(in_slot(i));
        s->bound_base = c0;
        s->bound_cycles = cc;
        if (gs_status st = sim_step(s, cc)) return st;
        CU(cudaEventRecord(ev_comp[i & 1], s->stream));
        if (host_out) {
            CU(cudaStreamWaitEvent(s->copy, ev_comp[i & 1], 0));
            CU(cudaMemcpyAsync(host_out + (size_t)i * chunk * p.n_po * w, out_slot(i), (size_t)cc * p.n_po * w * 8,
                               cudaMemcpyDeviceToHost, s->copy));
            CU(cudaEventRecord(ev_out[i & 1], s->copy));
        }
    }
    // detach the sink and the staging slot: a generated binding from before the call is
    // restored (the seed in Ctl is untouched by the streamed run), any other is cleared;
    // the sim's stream completes only after the last output copy
    if (prev_bound == 1) {
        CU(launch_set_binding(s->ctl(), 0ull, 0ull, 0u, 0ull, 0ull, 0ull, s->stream));
        s->bound = 1;
        s->bound_seed = prev_seed;
        s->bound_ptr = 0;
        s->bound_cycles = 0;
    } else {
        CU(launch_set_binding(s->ctl(), s->bound_ptr, s->bound_base, 1u, 0ull, 0ull, 0ull, s->stream));
        s->bound = 0;
    }
    CU(cudaEventRecord(ev_in[0], s->copy));
    CU(cudaStreamWaitEvent(s->stream, ev_in[0], 0));
    clear_error();
    return GS_OK;
}

static gs_status sim_read_outputs(gs_sim* s, uint64_t* host, size_t nwords) {
    if (gs_status st = check_sim(s, "gs_sim_read_outputs")) return st;
    const Program& p = *s->prog;
    const size_t need = (size_t)p.n_po * s->words;
    if (!host && need) return fail(GS_ERR_ARG, "gs_sim_read_outputs: NULL buffer");
    if (nwords < need) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_sim_read_outputs: need n_po * lanes/64 words");
    if (s->cycle == 0) return fail(GS_ERR_STATE, "gs_sim_read_outputs: no cycle stepped yet");
    CU(cudaSetDevice(s->opts.device));
    const uint32_t last_parity = (uint32_t)((s->cycle - 1) & 1);
    CU(launch_gather_rows(s->state(), s->stride, s->words, s->at<const uint32_t>(s->L.po_rows), p.n_po,
                          last_parity ? p.n_reg : 0, s->at<unsigned long long>(s->L.scratch), s->stream));
    if (need) CU(cudaMemcpyAsync(host, s->ws + s->L.scratch, need * 8, cudaMemcpyDeviceToHost, s->stream));
    CU(cudaStreamSynchronize(s->stream));
    clear_error();
    return GS_OK;
}

static gs_status sim_rw_registers(gs_sim* s, uint64_t* host_out, const uint64_t* host_in, size_t nwords) {
    const char* fn = host_out ? "gs_sim_read_registers" : "gs_sim_write_registers";
    if (gs_status st = check_sim(s, fn)) return st;
    const Program& p = *s->prog;
    const size_t need = (size_t)p.n_reg * s->words;
    if (!host_out && !host_in && need) return fail(GS_ERR_ARG, std::string(fn) + ": NULL buffer");
    if (nwords < need) return fail(GS_ERR_BUFFER_TOO_SMALL, std::string(fn) + ": need n_reg * lanes/64 words");
    CU(cudaSetDevice(s->opts.device));
    const uint32_t bank = (uint32_t)(s->cycle & 1);     // the bank the next cycle reads = Q(cycle)
    uint8_t* q = s->state() + (uint64_t)(p.row_q0 + bank * p.n_reg) * s->stride;
    if (need && host_out) CU(cudaMemcpyAsync(host_out, q, need * 8, cudaMemcpyDeviceToHost, s->stream));
    if (need && host_in) CU(cudaMemcpyAsync(q, host_in, need * 8, cudaMemcpyHostToDevice, s->stream));
    CU(cudaStreamSynchronize(s->stream));
    clear_error();
    return GS_OK;
}

static gs_status sim_read_trace(gs_sim* s, uint64_t* host, size_t nwords, uint32_t* cycles_recorded) {
    if (gs_status st = check_sim(s, "gs_sim_read_trace")) return st;
    const Program& p = *s->prog;
    const uint64_t rec = s->cycle < s->opts.trace_cycles ? s->cycle : s->opts.trace_cycles;
    const size_t need = (size_t)rec * p.n_po * s->opts.n_trace_words;
    if (!host && need) return fail(GS_ERR_ARG, "gs_sim_read_trace: NULL buffer");
    if (nwords < need) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_sim_read_trace: buffer too small");
    CU(cudaSetDevice(s->opts.device));
    if (need) CU(cudaMemcpyAsync(host, s->ws + s->L.trace, need * 8, cudaMemcpyDeviceToHost, s->stream));
    CU(cudaStreamSynchronize(s->stream));
    if (cycles_recorded) *cycles_recorded = (uint32_t)rec;
    clear_error();
    return GS_OK;
}

static gs_status compute_lane_sigs(gs_sim* s) {
    CU(cudaMemsetAsync(s->ws + s->L.ctl + offsetof(Ctl, sig_sum), 0, 8, s->stream));
    CU(launch_lane_sigs(s->ctl(), s->at<const unsigned long long>(s->L.misr) + (size_t)(s->cycle & 1) * 64 * s->words,
                        s->words, s->opts.lane_offset,
                        s->at<unsigned long long>(s->L.lane_sigs), s->stream));
    return GS_OK;
}

static gs_status sim_read_lane_signatures(gs_sim* s, uint64_t* host, size_t nlanes) {
    if (gs_status st = check_sim(s, "gs_sim_read_lane_signatures")) return st;
    if (!host) return fail(GS_ERR_ARG, "gs_sim_read_lane_signatures: NULL buffer");
    if (nlanes < s->opts.lanes) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_sim_read_lane_signatures: need `lanes` entries");
    CU(cudaSetDevice(s->opts.device));
    if (gs_status st = compute_lane_sigs(s)) return st;
    CU(cudaMemcpyAsync(host, s->ws + s->L.lane_sigs, (size_t)s->opts.lanes * 8, cudaMemcpyDeviceToHost, s->stream));
    CU(cudaStreamSynchronize(s->stream));
    clear_error();
    return GS_OK;
}

static gs_status sim_read_signature(gs_sim* s, gs_signature* out) {
    if (gs_status st = check_sim(s, "gs_sim_read_signature")) return st;
    if (!out) return fail(GS_ERR_ARG, "gs_sim_read_signature: NULL out");
    CU(cudaSetDevice(s->opts.device));
    if (gs_status st = compute_lane_sigs(s)) return st;
    Ctl h{};
    CU(cudaMemcpyAsync(&h, s->ctl(), sizeof(Ctl), cudaMemcpyDeviceToHost, s->stream));
    CU(cudaStreamSynchronize(s->stream));
    out->lane_sig_sum = h.sig_sum;
    out->out_popcount = h.popcount;
    out->ab_mismatch = h.ab_mismatch;
    out->invariant_violations = h.violations;
    out->cycles = h.cycle;
    clear_error();
    return GS_OK;
}

static uint64_t launches_per_cycle(const gs_sim* s) {
    const Program& p = *s->prog;
    if (s->opts.kernel == GS_KERNEL_TILE || s->opts.kernel == GS_KERNEL_CLUSTER)
        return 1;                                          // per gs_sim_step call, not per cycle
    uint64_t lv = 0;
    for (uint32_t l = 0; l < p.n_levels; ++l)
        if (p.level_off[l + 1] > p.level_off[l]) lv += s->lut_slabs > 1 && s->slabbed[l] ? s->lut_slabs : 1;
    const uint64_t per_level = s->opts.kernel == GS_KERNEL_AB ? 2 : 1;
    return (p.n_pi ? 1 : 0) + lv * per_level * s->groups + 1;
}

// level launches of one cycle (lane groups and the slab schedule included)
static uint64_t level_launches_per_cycle(const gs_sim* s) {
    const Program& p = *s->prog;
    uint64_t n = 0;
    for (uint32_t l = 0; l < p.n_levels; ++l)
        if (p.level_off[l + 1] > p.level_off[l])
            n += (uint64_t)s->groups * (s->lut_slabs > 1 && s->slabbed[l] ? s->lut_slabs : 1);
    return n;
}

static gs_status sim_profile_step(gs_sim* s, uint32_t n, gs_profile* out) {
    if (gs_status st = check_sim(s, "gs_sim_profile_step")) return st;
    if (!out) return fail(GS_ERR_ARG, "gs_sim_profile_step: NULL out");
    if (!s->bound) return fail(GS_ERR_STATE, "gs_sim_profile_step: no stimulus bound");
    if (s->bound == 2 && s->cycle + n > s->bound_base + s->bound_cycles)
        return fail(GS_ERR_STATE, "gs_sim_profile_step: stepping past the bound stimulus cycles");
    const Program& p = *s->prog;
    CU(cudaSetDevice(s->opts.device));
    // algorithmic bytes of a level: every gate reads k input rows, writes its output row,
    // plus the fused latch store (DESIGN.md §6 "algorithmic bytes")
    std::vector<double> lb(p.n_levels, 0.0);
    double all_bytes = 0;
    for (uint32_t l = 0; l < p.n_levels; ++l) {
        for (uint32_t g = p.level_off[l]; g < p.level_off[l + 1]; ++g)
            lb[l] += (double)(p.aux[g].k + 1 + (p.aux[g].qdst != NONE32 ? 1 : 0)) * (double)s->stride;
        all_bytes += lb[l];
    }
    std::memset(out, 0, sizeof(*out));
    if (s->opts.kernel == GS_KERNEL_TILE || s->opts.kernel == GS_KERNEL_CLUSTER) {
        // one launch runs all n cycles; "level" bytes are the same algorithmic gather model
        cudaEvent_t a0 = nullptr, a1 = nullptr;
        cudaError_t e = cudaEventCreate(&a0);
        if (e == cudaSuccess) e = cudaEventCreate(&a1);
        if (e == cudaSuccess) e = cudaEventRecord(a0, s->stream);
        if (e == cudaSuccess)
            e = s->opts.kernel == GS_KERNEL_TILE ? tile_launch(s, n, s->stream) : cluster_launch(s, n, s->stream);
        if (e == cudaSuccess) e = cudaEventRecord(a1, s->stream);
        if (e == cudaSuccess) e = cudaEventSynchronize(a1);
        float ms = 0;
        if (e == cudaSuccess) cudaEventElapsedTime(&ms, a0, a1);
        if (a0) cudaEventDestroy(a0);
        if (a1) cudaEventDestroy(a1);
        if (e != cudaSuccess) return fail(GS_ERR_CUDA, cudaGetErrorString(e));
        s->cycle += n;
        out->level_ms = ms;
        out->total_ms = ms;
        out->level_launches = n ? 1 : 0;
        out->total_launches = n ? 1 : 0;
        out->level_bytes = all_bytes * n;
        clear_error();
        return GS_OK;
    }
    std::vector<cudaEvent_t> evs(std::max<size_t>(2, 2 * (size_t)p.n_levels), nullptr);
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    cudaGraphExec_t px[2] = {nullptr, nullptr};
    struct Cleanup {
        std::vector<cudaEvent_t>& evs;
        cudaEvent_t &e0, &e1;
        cudaGraphExec_t* px;
        ~Cleanup() {
            for (auto& e : evs)
                if (e) cudaEventDestroy(e);
            if (e0) cudaEventDestroy(e0);
            if (e1) cudaEventDestroy(e1);
            for (int i = 0; i < 2; ++i)
                if (px[i]) cudaGraphExecDestroy(px[i]);
        }
    } cleanup{evs, e0, e1, px};
    for (auto& e : evs) CU(cudaEventCreate(&e));
    CU(cudaEventCreate(&e0));
    CU(cudaEventCreate(&e1));
    double level_ms = 0, total_ms = 0, level_bytes = 0;
    uint64_t lvl_launches = 0, launches = 0;
    const uint64_t per = launches_per_cycle(s);
    const uint64_t gs0 = s->grid_stride_launches, mg0 = s->multi_gate_launches;
    // concurrent lane groups: the branches only overlap as they do in gs_sim_step when the
    // cycle is replayed as its graph, so profile a graph of the cycle with timing-event
    // nodes at the fork and the join (eager launches of G x levels kernels would measure
    // the host's launch rate instead)
    auto prof_graph = [&](uint32_t parity) -> cudaError_t {
        if (px[parity]) return cudaSuccess;
        cudaGraph_t g = nullptr;
        cudaError_t e = cudaStreamBeginCapture(s->cap, cudaStreamCaptureModeThreadLocal);
        if (e != cudaSuccess) return e;
        e = cycle_launches(s, parity, s->cap, &evs, true);
        cudaError_t e2 = cudaStreamEndCapture(s->cap, &g);
        if (e == cudaSuccess) e = e2;
        if (e == cudaSuccess) e = cudaGraphInstantiate(&px[parity], g, 0);
        if (g) cudaGraphDestroy(g);
        return e;
    };
    for (uint32_t i = 0; i < n; ++i) {
        const uint32_t parity = (uint32_t)(s->cycle & 1);
        const bool region = s->groups > 1 || s->lut_slabs > 1;
        if (region) {
            CU(prof_graph(parity));
            CU(cudaEventRecord(e0, s->stream));
            CU(cudaGraphLaunch(px[parity], s->stream));
        } else {
            CU(cudaEventRecord(e0, s->stream));
            CU(cycle_launches(s, parity, s->stream, &evs));
        }
        CU(cudaEventRecord(e1, s->stream));
        s->cycle++;
        CU(cudaEventSynchronize(e1));
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        total_ms += ms;
        if (region) {                  // concurrent branches / slab runs cover every level
            cudaEventElapsedTime(&ms, evs[0], evs[1]);
            level_ms += ms;
            level_bytes += all_bytes;
            lvl_launches += level_launches_per_cycle(s);
        } else {
            for (uint32_t l = 0; l < p.n_levels; ++l) {
                if (p.level_off[l + 1] == p.level_off[l]) continue;
                cudaEventElapsedTime(&ms, evs[2 * (size_t)l], evs[2 * (size_t)l + 1]);
                level_ms += ms;
                level_bytes += lb[l];
                lvl_launches++;
            }
        }
        launches += per;
    }
    out->level_ms = level_ms;
    out->total_ms = total_ms;
    out->level_launches = lvl_launches;
    out->total_launches = launches;
    out->level_bytes = level_bytes;
    // launch decisions of the host side: with lane groups they were taken once per captured
    // graph (per parity), eagerly once per level launch otherwise
    out->grid_stride_launches = s->grid_stride_launches - gs0;
    out->multi_gate_launches = s->multi_gate_launches - mg0;
    clear_error();
    return GS_OK;
}

extern "C" {

gs_status gs_sim_workspace_bytes(const gs_program* prog, const gs_sim_opts* opts, size_t* bytes) {
    GS_TRY(return sim_workspace_bytes(prog, opts, bytes);)
}

gs_status gs_sim_create(const gs_program* prog, const gs_sim_opts* opts, void* dev_ws, size_t bytes, gs_sim** out) {
    GS_TRY(return sim_create(prog, opts, dev_ws, bytes, out);)
}

gs_status gs_sim_destroy(gs_sim* s) {
    if (!s) return GS_OK;
    GS_TRY({
        cudaSetDevice(s->opts.device);
        cudaStreamSynchronize(s->stream);
        free_sim(s);
        return GS_OK;
    })
}

gs_status gs_sim_reset(gs_sim* s) { GS_TRY(return sim_reset(s);) }

gs_status gs_sim_set_lane_offset(gs_sim* s, uint64_t lane_offset) { GS_TRY(return sim_set_lane_offset(s, lane_offset);) }

gs_status gs_sim_bind_stimulus_generated(gs_sim* s, uint64_t seed) { GS_TRY(return sim_bind_generated(s, seed);) }

gs_status gs_sim_bind_stimulus_device(gs_sim* s, const uint64_t* dev_words, uint32_t cycles) {
    GS_TRY(return sim_bind_device(s, dev_words, cycles);)
}

gs_status gs_sim_bind_stimulus_host(gs_sim* s, const uint64_t* words, uint32_t cycles) {
    GS_TRY(return sim_bind_host(s, words, cycles);)
}

gs_status gs_sim_step(gs_sim* s, uint32_t n) { GS_TRY(return sim_step(s, n);) }

gs_status gs_sim_run_streamed(gs_sim* s, const uint64_t* host_stim, uint64_t* host_out, uint32_t ncycles,
                              uint32_t chunk) {
    GS_TRY(return sim_run_streamed(s, host_stim, host_out, ncycles, chunk);)
}

gs_status gs_sim_sync(gs_sim* s) {
    GS_TRY({
        if (gs_status st = check_sim(s, "gs_sim_sync")) return st;
        CU(cudaSetDevice(s->opts.device));
        CU(cudaStreamSynchronize(s->stream));
        clear_error();
        return GS_OK;
    })
}

gs_status gs_sim_get_cycle(const gs_sim* s, uint64_t* cycle) {
    GS_TRY({
        if (!s || !cycle) return fail(GS_ERR_ARG, "gs_sim_get_cycle: NULL argument");
        *cycle = s->cycle;
        clear_error();
        return GS_OK;
    })
}

gs_status gs_sim_get_config(const gs_sim* s, int* kernel, uint32_t* lane_groups) {
    GS_TRY({
        if (!s || !kernel || !lane_groups) return fail(GS_ERR_ARG, "gs_sim_get_config: NULL argument");
        *kernel = s->opts.kernel;
        *lane_groups = s->groups;
        clear_error();
        return GS_OK;
    })
}

gs_status gs_sim_get_launch(const gs_sim* s, gs_launch_info* out) {
    GS_TRY({
        if (!s || !out) return fail(GS_ERR_ARG, "gs_sim_get_launch: NULL argument");
        std::memset(out, 0, sizeof(*out));
        out->kernel = s->opts.kernel;
        out->lane_groups = s->groups;
        out->tile_words = s->tw;
        out->tile_groups = s->opts.kernel == GS_KERNEL_TILE ? s->tile_groups : 0;
        out->tile_desc = (uint32_t)s->desc_smem;
        out->grid = s->opts.kernel == GS_KERNEL_TILE ? s->tile_grid
                    : s->opts.kernel == GS_KERNEL_CLUSTER ? s->clusters * s->cluster_size : 0;
        out->cluster_size = s->cluster_size;
        out->slab_lanes = s->opts.kernel == GS_KERNEL_CLUSTER ? s->slab_vec * 128
                          : s->lut_slabs > 1 ? s->lut_slab_vec * 128 : 0;
        out->live_slots = s->opts.kernel == GS_KERNEL_TILE ? s->tile.n_slots : 0;
        clear_error();
        return GS_OK;
    })
}

gs_status gs_sim_read_outputs(gs_sim* s, uint64_t* host, size_t nwords) { GS_TRY(return sim_read_outputs(s, host, nwords);) }

gs_status gs_sim_read_registers(gs_sim* s, uint64_t* host, size_t nwords) {
    GS_TRY(return sim_rw_registers(s, host, nullptr, nwords);)
}

gs_status gs_sim_write_registers(gs_sim* s, const uint64_t* host, size_t nwords) {
    GS_TRY({
        if (!host && s && s->prog->n_reg) return fail(GS_ERR_ARG, "gs_sim_write_registers: NULL buffer");
        return sim_rw_registers(s, nullptr, host, nwords);
    })
}

gs_status gs_sim_read_trace(gs_sim* s, uint64_t* host, size_t nwords, uint32_t* cycles_recorded) {
    GS_TRY(return sim_read_trace(s, host, nwords, cycles_recorded);)
}

gs_status gs_sim_read_lane_signatures(gs_sim* s, uint64_t* host, size_t nlanes) {
    GS_TRY(return sim_read_lane_signatures(s, host, nlanes);)
}

gs_status gs_sim_read_signature(gs_sim* s, gs_signature* out) { GS_TRY(return sim_read_signature(s, out);) }

gs_status gs_sim_launches_per_cycle(const gs_sim* s, uint64_t* launches) {
    GS_TRY({
        if (!s || !launches) return fail(GS_ERR_ARG, "gs_sim_launches_per_cycle: NULL argument");
        *launches = launches_per_cycle(s);
        clear_error();
        return GS_OK;
    })
}

gs_status gs_sim_profile_step(gs_sim* s, uint32_t n, gs_profile* out) { GS_TRY(return sim_profile_step(s, n, out);) }

}  // extern "C"
