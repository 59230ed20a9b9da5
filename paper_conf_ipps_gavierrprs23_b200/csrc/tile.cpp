// tile.cpp — shared-memory slot allocation for kernel T (kernels_tile.cu).
//
// Kernel T keeps the whole state of one lane tile in shared memory and runs every level
// of every cycle of a step for it (lanes are independent, so tiles never synchronise).
// Shared memory is small, so gate outputs do not get a row each: a gate's value occupies
// a slot from the level that produces it until the last level that reads it (the live
// range of the merged-layer neuron), and slots are reused greedily level by
// level (interval colouring; optimal for interval graphs).  Fixed slots: const0/const1,
// one per PI (rewritten each cycle), two banks of register slots (the double buffer of
// the recurrent connection).  Values read after the last level — primary outputs
// (MISR/trace) and register D nets not fused into the producing gate's store — live to
// the end of the cycle.
#include <algorithm>
#include <cstring>

#include "internal.h"

namespace gs {

gs_status tile_plan(const Program& p, TilePlan& t) {
    const uint32_t P = p.n_pi, R = p.n_reg, G = p.n_eval, D = p.n_levels;
    t = TilePlan();
    t.q0 = 2 + P;
    const uint32_t fixed = 2 + P + 2 * R;
    // row ref (state row, QFLAG for Q) -> which gate (exec index) it names, or NONE32
    auto gate_of = [&](uint32_t ref) -> uint32_t {
        if (ref & QFLAG) return NONE32;
        return ref >= p.row_gate0 ? ref - p.row_gate0 : NONE32;
    };
    // exec index -> level (1-based)
    std::vector<uint32_t> lvl(G);
    for (uint32_t l = 0; l < D; ++l)
        for (uint32_t g = p.level_off[l]; g < p.level_off[l + 1]; ++g) lvl[g] = l + 1;
    // last level reading each gate's value (D + 1 = read at the end of the cycle)
    std::vector<uint32_t> last(G, 0);
    auto use = [&](uint32_t ref, uint32_t at) {
        const uint32_t g = gate_of(ref);
        if (g != NONE32) last[g] = std::max(last[g], at);
    };
    for (uint32_t g = 0; g < G; ++g) {
        const uint32_t k = p.aux[g].k;
        for (uint32_t j = 0; j < k; ++j) use(j < 4 ? p.in_lo[(size_t)g * 4 + j] : p.in_hi[(size_t)g * 4 + j - 4], lvl[g]);
    }
    for (uint32_t r : p.po_rows) use(r, D + 1);
    for (uint32_t r : p.latch_src) use(r, D + 1);
    // greedy allocation, level by level: free slots whose last read is before this level
    std::vector<uint32_t> slot(G, NONE32);
    std::vector<std::vector<uint32_t>> expire(D + 2);
    std::vector<uint32_t> freelist;
    uint32_t n_slots = fixed;
    for (uint32_t l = 1; l <= D; ++l) {
        for (uint32_t g : expire[l - 1]) freelist.push_back(slot[g]);
        for (uint32_t g = p.level_off[l - 1]; g < p.level_off[l]; ++g) {
            uint32_t s;
            if (!freelist.empty()) { s = freelist.back(); freelist.pop_back(); }
            else s = n_slots++;
            slot[g] = s;
            // a value nobody reads (or only the fused latch store) is dead after its level
            expire[std::max(last[g], l)].push_back(g);
        }
    }
    if (n_slots > 65535) return fail(GS_ERR_ARG, "TILE: more than 65535 live slots");
    t.n_slots = n_slots;
    auto slot_of = [&](uint32_t ref) -> uint32_t {
        if (ref & QFLAG) return t.q0 + ((ref & ~QFLAG) - p.row_q0);   // bank-0 Q slot
        if (ref < p.row_gate0) return ref;                              // const / PI rows
        return slot[ref - p.row_gate0];
    };
    // descriptors (16 B): x = in0 | in1 << 16, y = in2 | in3 << 16, z = tt[15:0] | out << 16,
    // w = k | (fused-latch register + 1) << 4; gates with k > 4 add 3 x 16 B in desc_hi:
    // {in4 | in5 << 16, in6 | in7 << 16, 0, 0} and the whole 256-bit table
    t.desc.resize(G);
    t.desc_hi.assign(p.any_wide ? (size_t)G * 12 : 0, 0);
    for (uint32_t g = 0; g < G; ++g) {
        const uint32_t k = p.aux[g].k;
        uint32_t in[8] = {0, 0, 0, 0, 0, 0, 0, 0};   // unused inputs read const0 (slot 0)
        for (uint32_t j = 0; j < k; ++j)
            in[j] = slot_of(j < 4 ? p.in_lo[(size_t)g * 4 + j] : p.in_hi[(size_t)g * 4 + j - 4]);
        const uint64_t tt = p.aux[g].tt;
        TileDesc d;
        d.in01 = in[0] | (in[1] << 16);
        d.in23 = in[2] | (in[3] << 16);
        d.tt = (uint32_t)(tt & 0xFFFFu) | (slot[g] << 16);
        const uint32_t reg = p.aux[g].qdst == NONE32 ? 0 : p.aux[g].qdst - p.row_q0 + 1;
        d.kreg = k | (reg << 4);
        t.desc[g] = d;
        if (p.any_wide) {
            uint32_t* h = &t.desc_hi[(size_t)g * 12];
            h[0] = in[4] | (in[5] << 16);
            h[1] = in[6] | (in[7] << 16);
            for (uint32_t w = 0; w < 4; ++w) {
                const uint64_t word = p.tt_full.empty() ? (w ? 0 : tt) : p.tt_full[(size_t)g * 4 + w];
                h[4 + 2 * w] = (uint32_t)word;
                h[5 + 2 * w] = (uint32_t)(word >> 32);
            }
        }
    }
    if (p.max_k <= 2 && p.n_reg == 0 && !p.any_wide) {
        t.desc_n.resize((size_t)G * 2);
        for (uint32_t g = 0; g < G; ++g) {
            t.desc_n[2 * (size_t)g] = t.desc[g].in01;
            t.desc_n[2 * (size_t)g + 1] = t.desc[g].tt;
        }
    }
    for (uint32_t r : p.po_rows) t.po_slot.push_back(slot_of(r));
    for (size_t i = 0; i < p.latch_src.size(); ++i) {
        t.latch_src.push_back(slot_of(p.latch_src[i]));
        t.latch_dst.push_back(p.latch_dst[i]);
    }
    // writeback after a step: every PO's value goes to its state row (gs_sim_read_outputs
    // gathers PO rows); Q rows are written back from their slots directly.
    for (uint32_t o = 0; o < p.n_po; ++o) {
        const uint32_t r = p.po_rows[o];
        if (r & QFLAG) continue;                    // Q rows are written back anyway
        t.wb_row.push_back(r);
        t.wb_slot.push_back(slot_of(r));
    }
    return GS_OK;
}

}  // namespace gs
