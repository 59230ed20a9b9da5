// serialize.cpp — save / load a compiled program (gs_program_save / gs_program_load).
//
// The paper persists its compiled network as a model file (Fig. 1; Table I "Memory
// (MB)").  Here the compiled program — levels, descriptors, Möbius coefficients and
// kernel-B terms, register/output maps and the query tables — is written as a flat binary
// file: a fixed header (magic, format version, scalar fields, program_hash) followed by
// every vector as (uint64 element count, raw little-endian elements), then an FNV-1a
// checksum of the body.  Loading verifies the checksum, the table sizes and the program
// hash, so a truncated or edited file is rejected.
#include <cstdio>
#include <cstring>
#include <memory>
#include <string>

#include "internal.h"

namespace gs {

namespace {

constexpr char MAGIC[8] = {'G', 'S', 'I', 'M', 'P', 'R', 'G', '1'};
constexpr uint32_t FORMAT = 2;          // 2: no per-gate L2-hint table (0.2.0)

// FNV-1a over every byte of the file body (the trailing 8-byte checksum)
inline uint64_t fnv(uint64_t h, const void* p, size_t n) {
    const uint8_t* b = static_cast<const uint8_t*>(p);
    for (size_t i = 0; i < n; ++i) h = (h ^ b[i]) * 0x100000001B3ULL;
    return h;
}
constexpr uint64_t FNV0 = 0xCBF29CE484222325ULL;

struct Writer {
    FILE* f;
    bool ok = true;
    uint64_t sum = FNV0;
    void raw(const void* p, size_t n) {
        ok = ok && (n == 0 || fwrite(p, 1, n, f) == n);
        sum = fnv(sum, p, n);
    }
    template <class T> void pod(const T& v) { raw(&v, sizeof(T)); }
    template <class T> void vec(const std::vector<T>& v) {
        pod<uint64_t>(v.size());
        raw(v.data(), v.size() * sizeof(T));
    }
};

struct Reader {
    FILE* f;
    bool ok = true;
    uint64_t sum = FNV0;
    void raw(void* p, size_t n) {
        ok = ok && (n == 0 || fread(p, 1, n, f) == n);
        if (ok) sum = fnv(sum, p, n);
    }
    template <class T> void pod(T& v) { raw(&v, sizeof(T)); }
    template <class T> void vec(std::vector<T>& v) {
        uint64_t n = 0;
        pod(n);
        if (!ok || n > (1ull << 36) / sizeof(T)) { ok = false; return; }
        v.resize(n);
        raw(v.data(), n * sizeof(T));
    }
};

// Every index the device or the host planner dereferences, checked against the arrays it
// points into (a file with recomputed checksums must not reach a kernel with an out-of-range
// row, register or offset).  Returns an empty string when the program is consistent.
std::string validate(const Program& q) {
    auto bad = [](const std::string& m) { return m; };
    if (q.row_pi0 != 2 || q.row_q0 != 2 + q.n_pi || q.row_gate0 != q.row_q0 + 2 * q.n_reg ||
        q.n_rows != (uint64_t)q.row_gate0 + q.n_eval || q.n_rows >= QFLAG)
        return bad("row map");
    if (q.max_k > GS_MAX_K_POLY || q.n_eval > q.n_gates) return bad("sizes");
    if (q.level_off.size() != (size_t)q.n_levels + 1 || q.level_off[0] != 0 || q.level_off.back() != q.n_eval)
        return bad("level offsets");
    for (uint32_t l = 0; l < q.n_levels; ++l)
        if (q.level_off[l + 1] < q.level_off[l]) return bad("level offsets not monotonic");
    if (q.aux.size() != q.n_eval || q.in_lo.size() != (size_t)q.n_eval * 4 ||
        (q.any_wide && q.in_hi.size() != (size_t)q.n_eval * 4) || (!q.any_wide && !q.in_hi.empty()) ||
        (q.max_k > GS_MAX_K_LUT64 && q.tt_full.size() != (size_t)q.n_eval * 4) ||
        q.term_off.size() != (size_t)q.n_eval + 1 || q.exec_gate.size() != q.n_eval)
        return bad("descriptor table sizes");
    // a row ref is valid for a gate of level l when it names a constant / PI row, a bank-0 Q
    // row (with QFLAG), or a gate row of an EARLIER level (no race inside a level launch)
    auto ref_ok = [&](uint32_t ref, uint32_t gate_end) {
        if (ref & QFLAG) {
            const uint32_t r = ref & ~QFLAG;
            return r >= q.row_q0 && r < q.row_q0 + q.n_reg;
        }
        return ref < q.row_q0 || (ref >= q.row_gate0 && ref < (uint64_t)q.row_gate0 + gate_end);
    };
    for (uint32_t l = 0; l < q.n_levels; ++l)
        for (uint32_t g = q.level_off[l]; g < q.level_off[l + 1]; ++g) {
            const GateAux& a = q.aux[g];
            if (a.k < 1 || a.k > q.max_k || (a.k > 4 && !q.any_wide)) return bad("gate fan-in");
            if (a.k <= GS_MAX_K_LUT64 && a.k < 6 && (a.tt >> (1u << a.k)) != 0) return bad("truth-table bits");
            for (uint32_t j = 0; j < a.k; ++j) {
                const uint32_t ref = j < 4 ? q.in_lo[(size_t)g * 4 + j] : q.in_hi[(size_t)g * 4 + j - 4];
                if (!ref_ok(ref, q.level_off[l])) return bad("gate input row out of range");
            }
            if (a.qdst != NONE32 && (a.qdst < q.row_q0 || a.qdst >= q.row_q0 + q.n_reg)) return bad("latch register");
            if (q.term_off[g + 1] < q.term_off[g]) return bad("term offsets");
            if (q.exec_gate[g] >= q.n_gates) return bad("exec gate");
        }
    if (q.term_off[0] != 0 || q.term_off.back() != q.terms.size()) return bad("term offsets");
    for (uint32_t g = 0; g < q.n_eval; ++g)
        for (uint32_t t = q.term_off[g]; t < q.term_off[g + 1]; ++t)
            if ((q.terms[t] & 0xFFu) >= (1u << q.aux[g].k)) return bad("term monomial");
    if (q.po_rows.size() != q.n_po || q.reg_init.size() != q.n_reg || q.latch_src.size() != q.latch_dst.size())
        return bad("register / output map sizes");
    for (uint32_t r : q.po_rows)
        if (!ref_ok(r, q.n_eval)) return bad("output row out of range");
    for (size_t i = 0; i < q.latch_src.size(); ++i)
        if (!ref_ok(q.latch_src[i], q.n_eval) || q.latch_dst[i] >= q.n_reg) return bad("latch map");
    for (uint8_t v : q.reg_init)
        if (v > 1) return bad("register init");
    if (q.gate_level.size() != q.n_gates || q.coeff_off.size() != (size_t)q.n_gates + 1 ||
        q.lut_k.size() != q.n_gates || q.lut_in_off.size() != (size_t)q.n_gates + 1 ||
        q.lut_tt.size() != q.n_gates || (!q.lut_tt_hi.empty() && q.lut_tt_hi.size() != (size_t)q.n_gates * 3))
        return bad("query table sizes");
    if (q.coeff_off[0] != 0 || q.lut_in_off[0] != 0) return bad("query offsets");
    for (uint32_t g = 0; g < q.n_gates; ++g) {
        if (q.lut_k[g] > GS_MAX_K_POLY) return bad("query fan-in");
        if (q.coeff_off[g + 1] < q.coeff_off[g] || q.coeff_off[g + 1] - q.coeff_off[g] != (1u << q.lut_k[g]))
            return bad("coefficient offsets");
        if (q.lut_in_off[g + 1] < q.lut_in_off[g] || q.lut_in_off[g + 1] - q.lut_in_off[g] != q.lut_k[g])
            return bad("query input offsets");
    }
    if (q.coeffs.size() != q.coeff_off.back() || q.lut_in.size() != q.lut_in_off.back()) return bad("query arrays");
    if (q.info.n_eval_gates != q.n_eval || q.info.n_levels != q.n_levels || q.info.n_rows != q.n_rows ||
        q.info.n_pi != q.n_pi || q.info.n_reg != q.n_reg || q.info.n_po != q.n_po || q.info.n_gates != q.n_gates)
        return bad("info block");
    return std::string();
}

// every field of Program, in one order for both directions
template <class IO>
void fields(IO& io, Program& p) {
    io.pod(p.n_pi); io.pod(p.n_reg); io.pod(p.n_po); io.pod(p.n_gates); io.pod(p.n_eval); io.pod(p.n_levels);
    io.pod(p.row_pi0); io.pod(p.row_q0); io.pod(p.row_gate0); io.pod(p.n_rows);
    uint8_t wide = p.any_wide ? 1 : 0;
    io.pod(wide);
    p.any_wide = wide != 0;
    io.pod(p.max_k);
    io.vec(p.level_off); io.vec(p.in_lo); io.vec(p.in_hi); io.vec(p.aux); io.vec(p.tt_full);
    io.vec(p.term_off); io.vec(p.terms); io.vec(p.po_rows); io.vec(p.latch_src); io.vec(p.latch_dst);
    io.vec(p.reg_init); io.vec(p.gate_level); io.vec(p.coeff_off); io.vec(p.coeffs); io.vec(p.lut_k);
    io.vec(p.lut_in_off); io.vec(p.lut_in); io.vec(p.lut_tt); io.vec(p.lut_tt_hi); io.vec(p.exec_gate);
    io.pod(p.info);
}

}  // namespace
}  // namespace gs

using namespace gs;


static gs_status program_save(const gs_program* prog, const char* path) {
    if (!prog || !path) return fail(GS_ERR_ARG, "gs_program_save: NULL argument");
    FILE* f = fopen(path, "wb");
    if (!f) return fail(GS_ERR_ARG, std::string("gs_program_save: cannot open ") + path);
    Writer w{f};
    w.raw(MAGIC, sizeof(MAGIC));
    w.pod(FORMAT);
    fields(w, const_cast<Program&>(*prog->p));  // the writer only reads the fields
    const uint64_t sum = w.sum;
    w.pod(sum);
    const bool ok = w.ok && fclose(f) == 0;
    if (!ok) return fail(GS_ERR_ARG, std::string("gs_program_save: write failed: ") + path);
    clear_error();
    return GS_OK;
}

static gs_status program_load(const char* path, gs_program** out) {
    if (!path || !out) return fail(GS_ERR_ARG, "gs_program_load: NULL argument");
    FILE* f = fopen(path, "rb");
    if (!f) return fail(GS_ERR_ARG, std::string("gs_program_load: cannot open ") + path);
    Reader r{f};
    char magic[8];
    uint32_t format = 0;
    r.raw(magic, sizeof(magic));
    r.pod(format);
    if (!r.ok || std::memcmp(magic, MAGIC, sizeof(MAGIC)) != 0 || format != FORMAT) {
        fclose(f);
        return fail(GS_ERR_ARG, std::string("gs_program_load: not a gsim program file (or another format): ") + path);
    }
    std::unique_ptr<Program> p(new Program());
    uint64_t stored = 0, body = 0;
    try {
        fields(r, *p);
        body = r.sum;
        r.pod(stored);
    } catch (const std::bad_alloc&) {
        fclose(f);
        return fail(GS_ERR_NOMEM, "gs_program_load: out of host memory");
    }
    const int extra = fgetc(f);
    fclose(f);
    if (!r.ok || extra != EOF || stored != body)
        return fail(GS_ERR_ARG, std::string("gs_program_load: truncated or corrupt file (checksum): ") + path);
    // every index in range, then the program hash over the loaded descriptors
    const std::string why = validate(*p);
    if (!why.empty())
        return fail(GS_ERR_ARG, "gs_program_load: inconsistent program (" + why + "): " + path);
    if (program_hash(*p) != p->info.program_hash)
        return fail(GS_ERR_ARG, std::string("gs_program_load: inconsistent program (hash mismatch): ") + path);
    *out = new gs_program{p.release()};
    clear_error();
    return GS_OK;
}

extern "C" {

gs_status gs_program_save(const gs_program* prog, const char* path) { GS_TRY(return program_save(prog, path);) }

gs_status gs_program_load(const char* path, gs_program** out) { GS_TRY(return program_load(path, out);) }

}  // extern "C"
