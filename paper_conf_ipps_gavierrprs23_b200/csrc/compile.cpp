// compile.cpp — netlist -> levelized program (the "NN compiler" of PAPER.md §III-B..D).
//
//  * levelization: the merged NN layers of §III-D are the depth levels of
//    the LUT DAG: level(g) = 1 + max level of its gate inputs, PIs,
//    register Qs (pseudo-inputs) and constants at level 0.  One level = one
//    memory pass over the stimulus batch on the GPU (GPU time tracks #layers).
//  * balancing (optional): slack-based list scheduling within [ASAP, ALAP] keeps the
//    depth and flattens the level widths of unbalanced real circuits.
//  * TT -> multilinear coefficients: Algorithm 1 as an iterative
//    butterfly (one stage per variable), Eq. 1.
//  * row layout + per-level SoA descriptors for the device.
#include <algorithm>
#include <cstring>
#include <memory>
#include <queue>

#include "internal.h"

namespace gs {

// Algorithm 1 (LUTtoPoly): recursing on x_i splits the table into the
// halves with x_i = 0 / 1 and merges them as [w_left, w_right - w_left].  Doing the
// merge for one variable across the whole table is one butterfly stage; the stages
// for different variables act on different index bits and commute, so k stages give
// the same coefficients as the recursion (<= k 2^(k-1) subtractions).  Index
// bit i <-> x_i in S (LSB-first, reading R1).
void mobius_butterfly(const uint64_t* tt4, uint32_t k, int32_t* w) {
    const uint32_t n = 1u << k;
    for (uint32_t m = 0; m < n; ++m) w[m] = (int32_t)((tt4[m >> 6] >> (m & 63)) & 1u);
    for (uint32_t i = 0; i < k; ++i) {
        const uint32_t b = 1u << i;
        for (uint32_t m = 0; m < n; ++m)
            if (m & b) w[m] -= w[m ^ b];           // w_right - w_left
    }
}

static inline uint64_t hmix(uint64_t h, uint64_t v) {
    h ^= v + 0x9E3779B97F4A7C15ULL + (h << 6) + (h >> 2);
    return h * 0xff51afd7ed558ccdULL;
}

// Hash of everything the device evaluates (multi-rank consistency, program files): rows,
// levels, descriptors, tables, terms, register and output maps.
uint64_t program_hash(const Program& pr) {
    uint64_t h = hmix(0, pr.n_rows);
    h = hmix(h, ((uint64_t)pr.n_pi << 32) | pr.n_reg);
    for (uint32_t v : pr.level_off) h = hmix(h, v);
    for (uint32_t v : pr.in_lo) h = hmix(h, v);
    for (uint32_t v : pr.in_hi) h = hmix(h, v);
    for (uint64_t v : pr.tt_full) h = hmix(h, v);
    for (const GateAux& a : pr.aux) h = hmix(hmix(h, a.tt), ((uint64_t)a.qdst << 32) | a.k);
    for (uint32_t v : pr.terms) h = hmix(h, v);
    for (uint32_t v : pr.po_rows) h = hmix(h, v);
    for (size_t i = 0; i < pr.latch_src.size(); ++i) h = hmix(h, ((uint64_t)pr.latch_src[i] << 32) | pr.latch_dst[i]);
    for (uint8_t v : pr.reg_init) h = hmix(h, v);
    return h;
}

gs_status compile(const Netlist& nl, const gs_compile_opts& opts, Program*& out) {
    const uint32_t N = nl.n_nets();
    const uint32_t P = (uint32_t)nl.pi_net.size();
    const uint32_t R = (uint32_t)nl.reg_net.size();
    const uint32_t G = (uint32_t)nl.gate_net.size();
    const uint32_t O = (uint32_t)nl.po_net.size();

    // ---------------------------------------------------------------- validate
    for (uint32_t r = 0; r < R; ++r)
        if (nl.reg_d[r] == NONE32)
            return fail(GS_ERR_UNDRIVEN, "gs_compile: register " + std::to_string(r) + " has no D");
    for (uint32_t g = 0; g < G; ++g) {
        if (nl.gate_k[g] > opts.max_k)
            return fail(GS_ERR_ARITY, "gs_compile: gate " + std::to_string(g) + " has k > max_k");
        for (uint32_t e = nl.gate_in_off[g]; e < nl.gate_in_off[g + 1]; ++e)
            if (nl.gate_in[e] >= N)
                return fail(GS_ERR_ARG, "gs_compile: gate " + std::to_string(g) + " reads a missing net");
    }

    auto is_eval_gate_net = [&](uint32_t n) {
        return nl.net_kind[n] == NET_GATE && nl.gate_k[nl.net_index[n]] > 0;
    };

    // ---------------------------------------------------------------- gate DAG (Kahn)
    std::vector<uint32_t> indeg(G, 0), cons_off(G + 1, 0);
    for (uint32_t g = 0; g < G; ++g)
        for (uint32_t e = nl.gate_in_off[g]; e < nl.gate_in_off[g + 1]; ++e) {
            uint32_t n = nl.gate_in[e];
            if (is_eval_gate_net(n)) {
                indeg[g]++;
                cons_off[nl.net_index[n] + 1]++;
            }
        }
    for (uint32_t g = 0; g < G; ++g) cons_off[g + 1] += cons_off[g];
    std::vector<uint32_t> cons(cons_off[G]);
    {
        std::vector<uint32_t> fill(G, 0);
        for (uint32_t g = 0; g < G; ++g)
            for (uint32_t e = nl.gate_in_off[g]; e < nl.gate_in_off[g + 1]; ++e) {
                uint32_t n = nl.gate_in[e];
                if (is_eval_gate_net(n)) {
                    uint32_t p = nl.net_index[n];
                    cons[cons_off[p] + fill[p]++] = g;
                }
            }
    }
    std::vector<uint32_t> topo;
    topo.reserve(G);
    {
        std::vector<uint32_t> deg = indeg;
        for (uint32_t g = 0; g < G; ++g)
            if (deg[g] == 0) topo.push_back(g);
        for (size_t h = 0; h < topo.size(); ++h) {
            uint32_t g = topo[h];
            for (uint32_t e = cons_off[g]; e < cons_off[g + 1]; ++e)
                if (--deg[cons[e]] == 0) topo.push_back(cons[e]);
        }
        if (topo.size() != G)
            return fail(GS_ERR_COMB_LOOP, "gs_compile: combinational loop (" +
                                              std::to_string(G - topo.size()) + " gates on cycles)");
    }

    // ---------------------------------------------------------------- ASAP / ALAP
    std::vector<uint32_t> asap(G, 0), level(G, 0);
    uint32_t D = 0, n_eval = 0;
    for (uint32_t g : topo) {
        if (nl.gate_k[g] == 0) continue;               // constants are sources (level 0)
        n_eval++;
        uint32_t l = 0;
        for (uint32_t e = nl.gate_in_off[g]; e < nl.gate_in_off[g + 1]; ++e) {
            uint32_t n = nl.gate_in[e];
            if (is_eval_gate_net(n)) l = std::max(l, asap[nl.net_index[n]]);
        }
        asap[g] = l + 1;
        D = std::max(D, asap[g]);
    }
    std::vector<uint32_t> alap;
    if ((opts.balance || opts.level_seed) && n_eval > 0) {
        alap.assign(G, D);
        for (size_t i = topo.size(); i-- > 0;) {
            uint32_t g = topo[i];
            if (nl.gate_k[g] == 0) continue;
            uint32_t a = D;
            for (uint32_t e = cons_off[g]; e < cons_off[g + 1]; ++e) a = std::min(a, alap[cons[e]] - 1);
            alap[g] = a;
        }
    }
    // peak number of gate values live at one level boundary for a level assignment: a value
    // lives from its level to its last reader's level (outputs and leftover latch sources:
    // to the end of the cycle), the quantity tile.cpp's interval colouring allocates
    auto peak_live = [&](const std::vector<uint32_t>& lv) -> uint64_t {
        std::vector<int64_t> diff(D + 3, 0);
        std::vector<uint32_t> last(G, 0);
        for (uint32_t g = 0; g < G; ++g)
            if (nl.gate_k[g] > 0) last[g] = lv[g];
        for (uint32_t g = 0; g < G; ++g)
            for (uint32_t e = cons_off[g]; e < cons_off[g + 1]; ++e) last[g] = std::max(last[g], lv[cons[e]]);
        for (uint32_t o = 0; o < O; ++o) {
            const uint32_t n = nl.po_net[o];
            if (is_eval_gate_net(n)) last[nl.net_index[n]] = D + 1;
        }
        for (uint32_t r = 0; r < R; ++r) {
            const uint32_t n = nl.reg_d[r];
            if (is_eval_gate_net(n)) last[nl.net_index[n]] = D + 1;
        }
        for (uint32_t g = 0; g < G; ++g)
            if (nl.gate_k[g] > 0) {
                diff[lv[g]] += 1;
                diff[last[g] + 1] -= 1;
            }
        int64_t cur = 0, peak = 0;
        for (uint32_t l = 0; l < D + 3; ++l) peak = std::max(peak, cur += diff[l]);
        return (uint64_t)peak;
    };
    if (opts.level_seed && n_eval > 0) {
        // seeded random valid levels: in topological order, uniform in [1 + max input level,
        // ALAP]; the upper end stays >= the lower one because every input's level is <= its
        // own ALAP <= ALAP(g) - 1
        for (uint32_t g : topo) {
            if (nl.gate_k[g] == 0) continue;
            uint32_t lo = 1;
            for (uint32_t e = nl.gate_in_off[g]; e < nl.gate_in_off[g + 1]; ++e) {
                uint32_t n = nl.gate_in[e];
                if (is_eval_gate_net(n)) lo = std::max(lo, level[nl.net_index[n]] + 1);
            }
            uint64_t z = opts.level_seed ^ (0x9E3779B97F4A7C15ull * (g + 1));
            z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
            z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
            z ^= z >> 31;
            level[g] = lo + (uint32_t)(z % (uint64_t)(alap[g] - lo + 1));
        }
    } else if (opts.balance == 2 && n_eval > 0) {
        // ALAP: every gate as late as its consumers allow (same depth); a value is produced
        // right before it is needed, which shortens live ranges (kernel T's shared-memory
        // slots, tile.cpp) at the price of uneven widths
        level = alap;
    } else if (opts.balance && n_eval > 0) {
        // list scheduling, level by level: least slack (smallest ALAP) first, must place
        // every gate whose ALAP is this level, otherwise fill up to the mean width.
        const uint64_t target = (n_eval + D - 1) / D;
        typedef std::pair<uint64_t, uint32_t> Item;    // key = alap<<32 | asap, gate
        std::priority_queue<Item, std::vector<Item>, std::greater<Item>> ready;
        std::vector<uint32_t> deg = indeg;
        for (uint32_t g = 0; g < G; ++g)
            if (nl.gate_k[g] > 0 && deg[g] == 0) ready.push({((uint64_t)alap[g] << 32) | asap[g], g});
        std::vector<uint32_t> placed;
        for (uint32_t l = 1; l <= D; ++l) {
            placed.clear();
            while (!ready.empty()) {
                const Item it = ready.top();
                uint32_t a = (uint32_t)(it.first >> 32);
                if (placed.size() >= target && a > l) break;
                ready.pop();
                level[it.second] = l;
                placed.push_back(it.second);
            }
            for (uint32_t g : placed)
                for (uint32_t e = cons_off[g]; e < cons_off[g + 1]; ++e) {
                    uint32_t c = cons[e];
                    if (--deg[c] == 0) ready.push({((uint64_t)alap[c] << 32) | asap[c], c});
                }
        }
        if (!ready.empty()) return fail(GS_ERR_STATE, "gs_compile: internal balancing error");
        // Filling levels up to the mean width moves gates with large slack (the partial
        // products of a multiplier) early, where their values stay live for many levels.
        // Where ALAP levels hold markedly fewer values live at once (kernel T keeps every live
        // value of a tile in shared memory, so fewer live values = more lanes per SM), take ALAP
        // instead: C2 (32x32 multiplier) 752 -> 256 peak live values; synthetic circuits keep
        // the balanced levels (ALAP raises their peak).
        if (peak_live(level) * 4 > peak_live(alap) * 5) level = alap;
    } else {
        level = asap;
    }

    // ---------------------------------------------------------------- execution order
    std::unique_ptr<Program> p(new Program());   // freed on every early return / exception
    Program& pr = *p;
    pr.n_pi = P; pr.n_reg = R; pr.n_po = O; pr.n_gates = G; pr.n_eval = n_eval; pr.n_levels = D;
    pr.row_pi0 = 2;
    pr.row_q0 = 2 + P;
    pr.row_gate0 = 2 + P + 2 * R;
    pr.n_rows = (uint64_t)pr.row_gate0 + n_eval;
    if (pr.n_rows >= QFLAG) return fail(GS_ERR_ARG, "gs_compile: too many state rows");

    // counting sort by (level, k), stable in gate id
    pr.level_off.assign(D + 1, 0);
    std::vector<uint64_t> bucket((uint64_t)D * (GS_MAX_K_POLY + 1) + 1, 0);
    for (uint32_t g = 0; g < G; ++g)
        if (nl.gate_k[g] > 0) bucket[(uint64_t)(level[g] - 1) * (GS_MAX_K_POLY + 1) + nl.gate_k[g] + 1]++;
    for (size_t i = 1; i < bucket.size(); ++i) bucket[i] += bucket[i - 1];
    for (uint32_t l = 0; l <= D; ++l) pr.level_off[l] = (uint32_t)bucket[(uint64_t)l * (GS_MAX_K_POLY + 1)];
    std::vector<uint32_t> exec_pos(G, NONE32);
    pr.exec_gate.assign(n_eval, 0);
    for (uint32_t g = 0; g < G; ++g)
        if (nl.gate_k[g] > 0) {
            uint64_t b = (uint64_t)(level[g] - 1) * (GS_MAX_K_POLY + 1) + nl.gate_k[g];
            uint32_t pos = (uint32_t)bucket[b]++;
            exec_pos[g] = pos;
            pr.exec_gate[pos] = g;
        }

    auto row_of = [&](uint32_t n) -> uint32_t {
        uint32_t i = nl.net_index[n];
        switch (nl.net_kind[n]) {
            case NET_PI: return pr.row_pi0 + i;
            case NET_REG: return (pr.row_q0 + i) | QFLAG;
            default:
                if (nl.gate_k[i] == 0) return (uint32_t)(nl.gate_tt[i] & 1u);   // const0/const1 rows
                return pr.row_gate0 + exec_pos[i];
        }
    };

    // ---------------------------------------------------------------- descriptors
    pr.in_lo.assign((size_t)n_eval * 4, 0);
    pr.aux.resize(n_eval);
    for (uint32_t g = 0; g < G; ++g)
        if (nl.gate_k[g] > 4) pr.any_wide = true;
    if (pr.any_wide) pr.in_hi.assign((size_t)n_eval * 4, 0);
    for (uint32_t pos = 0; pos < n_eval; ++pos) {
        uint32_t g = pr.exec_gate[pos];
        uint32_t k = nl.gate_k[g];
        for (uint32_t j = 0; j < k; ++j) {
            uint32_t rr = row_of(nl.gate_in[nl.gate_in_off[g] + j]);
            if (j < 4) pr.in_lo[(size_t)pos * 4 + j] = rr;
            else pr.in_hi[(size_t)pos * 4 + (j - 4)] = rr;
        }
        pr.aux[pos].tt = nl.gate_tt[g];
        pr.max_k = std::max(pr.max_k, k);
        if (!nl.gate_tt_hi.empty()) {
            if (pr.tt_full.empty()) pr.tt_full.assign((size_t)n_eval * 4, 0);
            nl.table(g, &pr.tt_full[(size_t)pos * 4]);
        }
        pr.aux[pos].qdst = NONE32;
        pr.aux[pos].k = k;
    }
    // registers: fuse the latch into the D-driving gate's store when possible (the
    // recurrent connection of P:241 becomes a dual store into the other Q bank)
    pr.reg_init = nl.reg_init;
    for (uint32_t r = 0; r < R; ++r) {
        uint32_t d = nl.reg_d[r];
        if (is_eval_gate_net(d)) {
            uint32_t pos = exec_pos[nl.net_index[d]];
            if (pr.aux[pos].qdst == NONE32) {
                pr.aux[pos].qdst = pr.row_q0 + r;
                continue;
            }
        }
        pr.latch_src.push_back(row_of(d));
        pr.latch_dst.push_back(r);
    }
    pr.po_rows.resize(O);
    for (uint32_t o = 0; o < O; ++o) pr.po_rows[o] = row_of(nl.po_net[o]);

    pr.lut_k = nl.gate_k;
    pr.lut_in_off = nl.gate_in_off;
    pr.lut_in = nl.gate_in;
    pr.lut_tt = nl.gate_tt;
    pr.lut_tt_hi = nl.gate_tt_hi;

    // ---------------------------------------------------------------- coefficients
    pr.gate_level.assign(G, 0);
    pr.coeff_off.assign(G + 1, 0);
    for (uint32_t g = 0; g < G; ++g) {
        pr.gate_level[g] = nl.gate_k[g] ? level[g] : 0;
        pr.coeff_off[g + 1] = pr.coeff_off[g] + (1u << nl.gate_k[g]);
    }
    pr.coeffs.assign(pr.coeff_off[G], 0);
    for (uint32_t g = 0; g < G; ++g) {
        uint64_t t4[4];
        nl.table(g, t4);
        mobius_butterfly(t4, nl.gate_k[g], &pr.coeffs[pr.coeff_off[g]]);
    }
    pr.term_off.assign(n_eval + 1, 0);
    uint64_t nnz = 0, hidden = 0, edges = 0;
    for (uint32_t pos = 0; pos < n_eval; ++pos) {
        uint32_t g = pr.exec_gate[pos];
        uint32_t k = nl.gate_k[g];
        const int32_t* w = &pr.coeffs[pr.coeff_off[g]];
        for (uint32_t S = 0; S < (1u << k); ++S) {
            if (w[S] == 0) continue;
            // hidden neuron h_S: weights 1 on x_s (s in S), bias |S|-1 (Eq. 3);
            // output weight w_S
            uint32_t bias = (uint32_t)(__builtin_popcount(S) - 1) & 0xFFu;
            pr.terms.push_back(S | (bias << 8) | ((uint32_t)(uint16_t)(int16_t)w[S] << 16));
        }
        pr.term_off[pos + 1] = (uint32_t)pr.terms.size();
        nnz += pr.term_off[pos + 1] - pr.term_off[pos];
        hidden += 1ull << k;
        edges += k;
    }

    // ---------------------------------------------------------------- info + hash
    gs_program_info& in = pr.info;
    std::memset(&in, 0, sizeof(in));
    in.n_pi = P; in.n_reg = R; in.n_po = O; in.n_gates = G; in.n_eval_gates = n_eval;
    in.n_levels = D;
    in.min_width = D ? 0xFFFFFFFFu : 0;
    for (uint32_t l = 0; l < D; ++l) {
        uint32_t w = pr.level_off[l + 1] - pr.level_off[l];
        in.max_width = std::max(in.max_width, w);
        in.min_width = std::min(in.min_width, w);
    }
    for (uint32_t g = 0; g < G; ++g) in.k_hist[nl.gate_k[g]]++;
    in.n_edges = edges;
    in.nnz_coeffs = nnz;
    in.hidden_neurons = hidden;
    in.n_rows = pr.n_rows;
    in.program_hash = program_hash(pr);
    out = p.release();
    return GS_OK;
}

}  // namespace gs
