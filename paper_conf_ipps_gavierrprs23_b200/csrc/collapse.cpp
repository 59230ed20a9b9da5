// collapse.cpp — in-compiler cone collapsing into LUTs of at most L inputs.
//
// The paper maps a circuit into LUTs of at most L inputs before building the network
// (§III-B1, Fig. 3): L is the compiler's main hyperparameter — larger L
// gives fewer LUTs and a shallower graph (depth ~ O(1/log2 L)) at the price of 2^L-entry
// truth tables.  The paper uses ABC (a FlowMap variant) and a SAT solver; here the same
// step is a greedy, depth-driven cone collapse over the gate DAG with truth tables by
// enumeration (at most 2^L points per merge):
//   for every gate c in topological order, repeatedly absorb its deepest gate input g
//   while |inputs(c) \ {g} U inputs(g)| <= L; g stays alive while other consumers, a
//   primary output or a register still read it (duplication, as in FlowMap covers), and
//   dies — becomes an unreferenced k = 0 constant — when its last reader absorbed it.
// The collapsed netlist has the same nets (ids) and computes the same function of the
// PIs and register Qs on every net that is still read, so simulation results are
// identical (tested against the oracle on the original netlist).
#include <algorithm>
#include <array>
#include <vector>

#include "internal.h"

namespace gs {

gs_status collapse_luts(const Netlist& nl, uint32_t L, Netlist& out) {
    const uint32_t N = nl.n_nets(), G = (uint32_t)nl.gate_net.size();
    std::vector<std::vector<uint32_t>> ins(G);
    typedef std::array<uint64_t, 4> T4;                       // tables of up to 2^8 bits
    std::vector<T4> tt(G);
    for (uint32_t g = 0; g < G; ++g) nl.table(g, tt[g].data());
    auto bit = [](const T4& t, uint32_t m) -> uint32_t { return (uint32_t)((t[m >> 6] >> (m & 63)) & 1u); };
    for (uint32_t g = 0; g < G; ++g) {
        ins[g].assign(nl.gate_in.begin() + nl.gate_in_off[g], nl.gate_in.begin() + nl.gate_in_off[g + 1]);
        for (uint32_t n : ins[g])
            if (n >= N) return fail(GS_ERR_ARG, "gs_compile: gate " + std::to_string(g) + " reads a missing net");
    }
    auto gate_of = [&](uint32_t n) -> uint32_t {
        return nl.net_kind[n] == NET_GATE ? nl.net_index[n] : NONE32;
    };
    // topological order of the gate DAG (Kahn; registers cut)
    std::vector<uint32_t> indeg(G, 0), order;
    std::vector<std::vector<uint32_t>> users(G);
    for (uint32_t g = 0; g < G; ++g)
        for (uint32_t n : ins[g]) {
            const uint32_t p = gate_of(n);
            if (p != NONE32) { indeg[g]++; users[p].push_back(g); }
        }
    for (uint32_t g = 0; g < G; ++g)
        if (!indeg[g]) order.push_back(g);
    for (size_t h = 0; h < order.size(); ++h)
        for (uint32_t u : users[order[h]])
            if (--indeg[u] == 0) order.push_back(u);
    if (order.size() != G) return fail(GS_ERR_COMB_LOOP, "gs_compile: combinational loop");
    // readers of every net: distinct consumer gates + primary outputs + register D
    std::vector<uint32_t> readers(N, 0), pinned(N, 0);
    auto distinct = [](std::vector<uint32_t> v) {
        std::sort(v.begin(), v.end());
        v.erase(std::unique(v.begin(), v.end()), v.end());
        return v;
    };
    for (uint32_t g = 0; g < G; ++g)
        for (uint32_t n : distinct(ins[g])) readers[n]++;
    for (uint32_t n : nl.po_net) pinned[n] = 1;
    for (uint32_t d : nl.reg_d)
        if (d != NONE32) pinned[d] = 1;
    std::vector<uint8_t> dead(G, 0);
    std::vector<uint32_t> level(N, 0);
    // kill a gate nobody reads any more; its inputs lose a reader (cascades upstream)
    std::vector<uint32_t> stack;
    auto release = [&](uint32_t n) {
        stack.push_back(n);
        while (!stack.empty()) {
            const uint32_t m = stack.back();
            stack.pop_back();
            if (--readers[m] || pinned[m]) continue;
            const uint32_t g = gate_of(m);
            if (g == NONE32 || dead[g]) continue;
            dead[g] = 1;
            for (uint32_t x : distinct(ins[g])) stack.push_back(x);
            ins[g].clear();
            tt[g] = T4{0, 0, 0, 0};
        }
    };
    for (uint32_t c : order) {
        if (ins[c].empty()) continue;                          // constant
        for (;;) {
            // deepest absorbable gate input
            uint32_t best = NONE32, best_lv = 0;
            std::vector<uint32_t> best_merged;
            for (uint32_t n : distinct(ins[c])) {
                const uint32_t g = gate_of(n);
                if (g == NONE32 || dead[g] || ins[g].empty()) continue;
                std::vector<uint32_t> m;
                for (uint32_t x : ins[c])
                    if (x != n) m.push_back(x);
                m.insert(m.end(), ins[g].begin(), ins[g].end());
                m = distinct(m);
                if (m.size() > L) continue;
                if (best == NONE32 || level[n] > best_lv) { best = g; best_lv = level[n]; best_merged = m; }
            }
            if (best == NONE32) break;
            // compose: new table over best_merged (bit j of the point = value of net best_merged[j])
            const uint32_t gnet = nl.gate_net[best];
            const std::vector<uint32_t>& gi = ins[best];
            const uint32_t K = (uint32_t)best_merged.size();
            T4 nt{0, 0, 0, 0};
            for (uint32_t m = 0; m < (1u << K); ++m) {
                auto val = [&](uint32_t net) -> uint32_t {
                    const size_t j = std::lower_bound(best_merged.begin(), best_merged.end(), net) - best_merged.begin();
                    return (m >> j) & 1u;
                };
                uint32_t gx = 0;
                for (size_t i = 0; i < gi.size(); ++i) gx |= val(gi[i]) << i;
                const uint32_t gv = bit(tt[best], gx);
                uint32_t cx = 0;
                for (size_t i = 0; i < ins[c].size(); ++i) cx |= (ins[c][i] == gnet ? gv : val(ins[c][i])) << i;
                nt[m >> 6] |= (uint64_t)bit(tt[c], cx) << (m & 63);
            }
            // reader bookkeeping: c now reads best_merged instead of its old inputs
            const std::vector<uint32_t> old = distinct(ins[c]);
            for (uint32_t x : best_merged)
                if (!std::binary_search(old.begin(), old.end(), x)) readers[x]++;
            ins[c] = best_merged;
            tt[c] = nt;
            release(gnet);                                     // c no longer reads g
        }
        uint32_t lv = 0;
        for (uint32_t n : ins[c]) lv = std::max(lv, level[n]);
        level[nl.gate_net[c]] = lv + 1;
    }
    // rebuild the netlist: same nets, dead gates become unreferenced k = 0 constants
    out = nl;
    out.gate_k.assign(G, 0);
    out.gate_in_off.assign(G + 1, 0);
    out.gate_in.clear();
    bool wide = false;
    for (uint32_t g = 0; g < G; ++g) wide = wide || ins[g].size() > GS_MAX_K;
    out.gate_tt_hi.assign(wide ? (size_t)G * 3 : 0, 0);
    for (uint32_t g = 0; g < G; ++g) {
        out.gate_k[g] = (uint8_t)ins[g].size();
        out.gate_in.insert(out.gate_in.end(), ins[g].begin(), ins[g].end());
        out.gate_in_off[g + 1] = (uint32_t)out.gate_in.size();
        out.gate_tt[g] = dead[g] ? 0 : tt[g][0];
        if (wide && !dead[g])
            for (int j = 0; j < 3; ++j) out.gate_tt_hi[(size_t)g * 3 + j] = tt[g][1 + j];
    }
    return GS_OK;
}

}  // namespace gs
