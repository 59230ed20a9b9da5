// netlist.cpp — error state and the netlist half of the C-ABI (include/gsim.h).
//
// A netlist is the computation graph of PAPER.md P:167 (§III-B1): nodes are binary
// signals, every LUT node has at most L predecessors, plus the D flip-flops of
// P:236-241 (§III-C) whose Q is a pseudo-input and whose D is a pseudo-output.
#include <cstring>
#include <memory>
#include <new>

#include "internal.h"

namespace gs {
static thread_local std::string g_err;
void set_error(const std::string& msg) {
    try {
        g_err = msg;
    } catch (...) {                   // out of memory for the message: keep the code only
        g_err.clear();
    }
}
void clear_error() { g_err.clear(); }
gs_status fail(gs_status code, const std::string& msg) {
    set_error(msg);
    return code;
}
}  // namespace gs

using namespace gs;

struct gs_netlist {
    Netlist nl;
};


extern "C" {

const char* gs_last_error(void) { return g_err.c_str(); }
const char* gs_version(void) { return GSIM_VERSION; }
#ifndef GS_BUILD_ID
#define GS_BUILD_ID "unknown"
#endif
const char* gs_build_id(void) { return GS_BUILD_ID; }

gs_status gs_netlist_create(gs_netlist** out) {
    if (!out) return fail(GS_ERR_ARG, "gs_netlist_create: out is NULL");
    GS_TRY(*out = new gs_netlist(); clear_error(); return GS_OK;)
}

gs_status gs_netlist_destroy(gs_netlist* nl) {
    GS_TRY(delete nl; return GS_OK;)
}

static uint32_t new_net(Netlist& n, NetKind kind, uint32_t index) {
    n.net_kind.push_back(kind);
    n.net_index.push_back(index);
    return n.n_nets() - 1;
}

gs_status gs_add_input(gs_netlist* h, gs_net* out) {
    if (!h || !out) return fail(GS_ERR_ARG, "gs_add_input: NULL argument");
    GS_TRY({
        Netlist& n = h->nl;
        uint32_t id = new_net(n, NET_PI, (uint32_t)n.pi_net.size());
        n.pi_net.push_back(id);
        *out = id;
        clear_error();
        return GS_OK;
    })
}

gs_status gs_add_gate(gs_netlist* h, uint32_t k, const gs_net* in, uint64_t tt, gs_net* out) {
    GS_TRY(
        if (!h || !out || (k && !in)) return fail(GS_ERR_ARG, "gs_add_gate: NULL argument");
        if (k > GS_MAX_K) return fail(GS_ERR_ARITY, "gs_add_gate: k > GS_MAX_K");
        if (k < 6 && (tt >> (1u << k)) != 0)
            return fail(GS_ERR_ARG, "gs_add_gate: truth-table bits >= 2^k must be zero");
        GS_TRY({
            Netlist& n = h->nl;
            uint32_t id = new_net(n, NET_GATE, (uint32_t)n.gate_net.size());
            // inputs may name nets created later (checked at compile time)
            n.gate_net.push_back(id);
            n.gate_k.push_back((uint8_t)k);
            for (uint32_t i = 0; i < k; ++i) n.gate_in.push_back(in[i]);
            n.gate_in_off.push_back((uint32_t)n.gate_in.size());
            n.gate_tt.push_back(tt);
            if (!n.gate_tt_hi.empty()) n.gate_tt_hi.insert(n.gate_tt_hi.end(), 3, 0);
            *out = id;
            clear_error();
            return GS_OK;
        })
    )
}

gs_status gs_add_gate_wide(gs_netlist* h, uint32_t k, const gs_net* in, const uint64_t* tt_words, gs_net* out) {
    GS_TRY(
        if (!h || !out || (k && !in) || !tt_words) return fail(GS_ERR_ARG, "gs_add_gate_wide: NULL argument");
        if (k > GS_MAX_K_POLY) return fail(GS_ERR_ARITY, "gs_add_gate_wide: k > GS_MAX_K_POLY");
        if (k <= GS_MAX_K) return gs_add_gate(h, k, in, tt_words[0], out);
        GS_TRY({
            Netlist& n = h->nl;
            const uint32_t words = (1u << k) / 64;
            gs_status st = gs_add_gate(h, 0, nullptr, 0, out);   // allocate the net, then fill it in
            if (st != GS_OK) return st;
            n.gate_tt_hi.resize(n.gate_tt.size() * 3, 0);       // from now on 3 words per gate
            const uint32_t g = (uint32_t)n.gate_net.size() - 1;
            n.gate_k[g] = (uint8_t)k;                              // k = 0 pushed no inputs
            for (uint32_t i = 0; i < k; ++i) n.gate_in.push_back(in[i]);
            n.gate_in_off[g + 1] = (uint32_t)n.gate_in.size();
            n.gate_tt[g] = tt_words[0];
            for (uint32_t j = 1; j < 4; ++j) n.gate_tt_hi[(size_t)g * 3 + j - 1] = j < words ? tt_words[j] : 0;
            clear_error();
            return GS_OK;
        })
    )
}

gs_status gs_add_const(gs_netlist* h, int value, gs_net* out) {
    GS_TRY(
        if (value != 0 && value != 1) return fail(GS_ERR_ARG, "gs_add_const: value must be 0 or 1");
        return gs_add_gate(h, 0, nullptr, (uint64_t)value, out);
    )
}

gs_status gs_add_register(gs_netlist* h, int init, gs_net* q_out) {
    if (!h || !q_out) return fail(GS_ERR_ARG, "gs_add_register: NULL argument");
    if (init != 0 && init != 1) return fail(GS_ERR_ARG, "gs_add_register: init must be 0 or 1");
    GS_TRY({
        Netlist& n = h->nl;
        uint32_t id = new_net(n, NET_REG, (uint32_t)n.reg_net.size());
        n.reg_net.push_back(id);
        n.reg_init.push_back((uint8_t)init);
        n.reg_d.push_back(NONE32);
        *q_out = id;
        clear_error();
        return GS_OK;
    })
}

gs_status gs_set_register_d(gs_netlist* h, gs_net q, gs_net d) {
    GS_TRY(
        if (!h) return fail(GS_ERR_ARG, "gs_set_register_d: NULL netlist");
        Netlist& n = h->nl;
        if (q >= n.n_nets() || n.net_kind[q] != NET_REG)
            return fail(GS_ERR_ARG, "gs_set_register_d: q is not a register net");
        if (d >= n.n_nets()) return fail(GS_ERR_ARG, "gs_set_register_d: d is not an existing net");
        n.reg_d[n.net_index[q]] = d;
        clear_error();
        return GS_OK;
    )
}

gs_status gs_mark_output(gs_netlist* h, gs_net net, uint32_t* po_index) {
    GS_TRY(
        if (!h) return fail(GS_ERR_ARG, "gs_mark_output: NULL netlist");
        Netlist& n = h->nl;
        if (net >= n.n_nets()) return fail(GS_ERR_ARG, "gs_mark_output: not an existing net");
        GS_TRY({
            n.po_net.push_back(net);
            if (po_index) *po_index = (uint32_t)n.po_net.size() - 1;
            clear_error();
            return GS_OK;
        })
    )
}

gs_status gs_netlist_load_arrays(gs_netlist* h, const gs_netlist_arrays* a) {
    GS_TRY(
        if (!h || !a) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: NULL argument");
        Netlist& n = h->nl;
        if (n.n_nets() != 0 || !n.po_net.empty())
            return fail(GS_ERR_STATE, "gs_netlist_load_arrays: netlist is not empty");
        if ((a->n_reg && (!a->reg_init || !a->reg_d)) || (a->n_gates && (!a->gate_k || !a->gate_in_off ||
            !a->gate_tt)) || (a->n_po && !a->po))
            return fail(GS_ERR_ARG, "gs_netlist_load_arrays: NULL array");
        uint64_t N = (uint64_t)a->n_pi + a->n_reg + a->n_gates;
        if (N >= (uint64_t)QFLAG) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: too many nets");
        if (a->n_gates && a->gate_in_off[0] != 0)
            return fail(GS_ERR_ARG, "gs_netlist_load_arrays: gate_in_off[0] must be 0");
        for (uint32_t g = 0; g < a->n_gates; ++g) {
            uint32_t k = a->gate_k[g];
            if (k > GS_MAX_K_POLY) return fail(GS_ERR_ARITY, "gs_netlist_load_arrays: gate with k > GS_MAX_K_POLY");
            if (k > GS_MAX_K && !a->gate_tt_hi)
                return fail(GS_ERR_ARG, "gs_netlist_load_arrays: gates with k > 6 need gate_tt_hi");
            if (a->gate_in_off[g + 1] != a->gate_in_off[g] + k)
                return fail(GS_ERR_ARG, "gs_netlist_load_arrays: gate_in_off inconsistent with gate_k");
            if (k < 6 && (a->gate_tt[g] >> (1u << k)) != 0)
                return fail(GS_ERR_ARG, "gs_netlist_load_arrays: truth-table bits >= 2^k must be zero");
        }
        uint64_t E = a->n_gates ? a->gate_in_off[a->n_gates] : 0;
        if (E && !a->gate_in) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: NULL gate_in");
        for (uint64_t e = 0; e < E; ++e)
            if (a->gate_in[e] >= N) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: gate input net out of range");
        for (uint32_t r = 0; r < a->n_reg; ++r) {
            if (a->reg_d[r] >= N) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: reg_d out of range");
            if (a->reg_init[r] > 1) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: reg_init must be 0/1");
        }
        for (uint32_t o = 0; o < a->n_po; ++o)
            if (a->po[o] >= N) return fail(GS_ERR_ARG, "gs_netlist_load_arrays: po out of range");
        GS_TRY({
            n.net_kind.resize(N);
            n.net_index.resize(N);
            n.pi_net.resize(a->n_pi);
            for (uint32_t p = 0; p < a->n_pi; ++p) {
                n.net_kind[p] = NET_PI; n.net_index[p] = p; n.pi_net[p] = p;
            }
            n.reg_net.resize(a->n_reg);
            for (uint32_t r = 0; r < a->n_reg; ++r) {
                uint32_t id = a->n_pi + r;
                n.net_kind[id] = NET_REG; n.net_index[id] = r; n.reg_net[r] = id;
            }
            n.reg_init.assign(a->reg_init, a->reg_init + a->n_reg);
            n.reg_d.assign(a->reg_d, a->reg_d + a->n_reg);
            n.gate_net.resize(a->n_gates);
            uint32_t gb = a->n_pi + a->n_reg;
            for (uint32_t g = 0; g < a->n_gates; ++g) {
                n.net_kind[gb + g] = NET_GATE; n.net_index[gb + g] = g; n.gate_net[g] = gb + g;
            }
            n.gate_k.assign(a->gate_k, a->gate_k + a->n_gates);
            n.gate_in_off.assign(a->gate_in_off, a->gate_in_off + a->n_gates + 1);
            if (a->n_gates == 0) n.gate_in_off.assign(1, 0);
            n.gate_in.assign(a->gate_in, a->gate_in + E);
            n.gate_tt.assign(a->gate_tt, a->gate_tt + a->n_gates);
            n.gate_tt_hi.clear();
            bool wide = false;
            for (uint32_t g = 0; g < a->n_gates && !wide; ++g) wide = a->gate_k[g] > GS_MAX_K;
            if (wide) {
                n.gate_tt_hi.assign(a->gate_tt_hi, a->gate_tt_hi + (size_t)a->n_gates * 3);
                for (uint32_t g = 0; g < a->n_gates; ++g)        // bits beyond 2^k must not leak in
                    for (uint32_t j = 0; j < 3; ++j)
                        if (a->gate_k[g] < 7 || (j + 1) * 64 >= (1u << a->gate_k[g])) n.gate_tt_hi[(size_t)g * 3 + j] = 0;
            }
            n.po_net.assign(a->po, a->po + a->n_po);
            clear_error();
            return GS_OK;
        })
    )
}

gs_status gs_netlist_get_counts(const gs_netlist* h, gs_netlist_counts* out) {
    GS_TRY(
        if (!h || !out) return fail(GS_ERR_ARG, "gs_netlist_get_counts: NULL argument");
        const Netlist& n = h->nl;
        out->n_nets = n.n_nets();
        out->n_pi = (uint32_t)n.pi_net.size();
        out->n_reg = (uint32_t)n.reg_net.size();
        out->n_gates = (uint32_t)n.gate_net.size();
        out->n_po = (uint32_t)n.po_net.size();
        out->n_edges = n.gate_in.size();
        clear_error();
        return GS_OK;
    )
}

// ------------------------------------------------------------------ compile front
gs_status gs_compile(const gs_netlist* h, const gs_compile_opts* opts, gs_program** out) {
    GS_TRY(
        NvtxRange nvtx("gs_compile");
        if (!h || !out) return fail(GS_ERR_ARG, "gs_compile: NULL argument");
        gs_compile_opts o{1, 0, 0, 0};
        if (opts) o = *opts;
        if (o.max_k == 0 || o.max_k > GS_MAX_K_POLY) o.max_k = GS_MAX_K_POLY;
        if (o.lut_k == 1 || o.lut_k > o.max_k)
            return fail(GS_ERR_ARG, "gs_compile: lut_k must be 0 or in [2, max_k]");
        Program* p = nullptr;
        gs_status st;
        try {
            if (o.lut_k) {
                Netlist collapsed;
                st = collapse_luts(h->nl, o.lut_k, collapsed);
                if (st == GS_OK) st = compile(collapsed, o, p);
            } else {
                st = compile(h->nl, o, p);
            }
        } catch (const std::bad_alloc&) {
            return fail(GS_ERR_NOMEM, "gs_compile: out of host memory");
        }
        std::unique_ptr<Program> owned(p);
        if (st != GS_OK) return st;
        *out = new gs_program{owned.get()};
        owned.release();
        clear_error();
        return GS_OK;
    )
}

gs_status gs_program_destroy(gs_program* prog) {
    GS_TRY(
        if (prog) {
            delete prog->p;
            delete prog;
        }
        return GS_OK;
    )
}

gs_status gs_program_get_info(const gs_program* prog, gs_program_info* out) {
    GS_TRY(
        if (!prog || !out) return fail(GS_ERR_ARG, "gs_program_get_info: NULL argument");
        *out = prog->p->info;
        clear_error();
        return GS_OK;
    )
}

gs_status gs_program_level_widths(const gs_program* prog, uint32_t* widths, uint32_t n) {
    GS_TRY(
        if (!prog || (!widths && n)) return fail(GS_ERR_ARG, "gs_program_level_widths: NULL argument");
        const Program& p = *prog->p;
        if (n < p.n_levels) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_program_level_widths: n < n_levels");
        for (uint32_t l = 0; l < p.n_levels; ++l) widths[l] = p.level_off[l + 1] - p.level_off[l];
        clear_error();
        return GS_OK;
    )
}

gs_status gs_program_gate_levels(const gs_program* prog, uint32_t* level, uint32_t n) {
    GS_TRY(
        if (!prog || (!level && n)) return fail(GS_ERR_ARG, "gs_program_gate_levels: NULL argument");
        const Program& p = *prog->p;
        if (n < p.n_gates) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_program_gate_levels: n < n_gates");
        std::memcpy(level, p.gate_level.data(), sizeof(uint32_t) * p.n_gates);
        clear_error();
        return GS_OK;
    )
}

gs_status gs_program_coeffs(const gs_program* prog, uint32_t gate, int32_t* w, uint32_t n) {
    GS_TRY(
        if (!prog || !w) return fail(GS_ERR_ARG, "gs_program_coeffs: NULL argument");
        const Program& p = *prog->p;
        if (gate >= p.n_gates) return fail(GS_ERR_ARG, "gs_program_coeffs: gate out of range");
        uint32_t cnt = p.coeff_off[gate + 1] - p.coeff_off[gate];
        if (n < cnt) return fail(GS_ERR_BUFFER_TOO_SMALL, "gs_program_coeffs: n < 2^k");
        std::memcpy(w, p.coeffs.data() + p.coeff_off[gate], sizeof(int32_t) * cnt);
        clear_error();
        return GS_OK;
    )
}

gs_status gs_program_gate_lut(const gs_program* prog, uint32_t gate, uint32_t* k, gs_net* in, uint64_t* tt) {
    GS_TRY(
        if (!prog || !k || !in || !tt) return fail(GS_ERR_ARG, "gs_program_gate_lut: NULL argument");
        const Program& p = *prog->p;
        if (gate >= p.n_gates) return fail(GS_ERR_ARG, "gs_program_gate_lut: gate out of range");
        *k = p.lut_k[gate];
        for (uint32_t j = 0; j < *k; ++j) in[j] = p.lut_in[p.lut_in_off[gate] + j];
        tt[0] = p.lut_tt[gate];
        for (uint32_t j = 0; j < 3; ++j) tt[1 + j] = p.lut_tt_hi.empty() ? 0 : p.lut_tt_hi[(size_t)gate * 3 + j];
        clear_error();
        return GS_OK;
    )
}

gs_status gs_program_tile_slots(const gs_program* prog, uint32_t* slots) {
    GS_TRY(
        if (!prog || !slots) return fail(GS_ERR_ARG, "gs_program_tile_slots: NULL argument");
        TilePlan t;
        if (gs_status st = tile_plan(*prog->p, t)) return st;
        *slots = t.n_slots;
        clear_error();
        return GS_OK;
    )
}

}  // extern "C"
