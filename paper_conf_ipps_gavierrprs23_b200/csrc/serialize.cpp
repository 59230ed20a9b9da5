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
constexpr uint32_t FORMAT = 1;

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

// every field of Program, in one order for both directions
template <class IO>
void fields(IO& io, Program& p) {
    io.pod(p.n_pi); io.pod(p.n_reg); io.pod(p.n_po); io.pod(p.n_gates); io.pod(p.n_eval); io.pod(p.n_levels);
    io.pod(p.row_pi0); io.pod(p.row_q0); io.pod(p.row_gate0); io.pod(p.n_rows);
    uint8_t wide = p.any_wide ? 1 : 0;
    io.pod(wide);
    p.any_wide = wide != 0;
    io.pod(p.max_k);
    io.vec(p.level_off); io.vec(p.in_lo); io.vec(p.in_hi); io.vec(p.aux); io.vec(p.hot); io.vec(p.tt_full);
    io.vec(p.term_off); io.vec(p.terms); io.vec(p.po_rows); io.vec(p.latch_src); io.vec(p.latch_dst);
    io.vec(p.reg_init); io.vec(p.gate_level); io.vec(p.coeff_off); io.vec(p.coeffs); io.vec(p.lut_k);
    io.vec(p.lut_in_off); io.vec(p.lut_in); io.vec(p.lut_tt); io.vec(p.lut_tt_hi); io.vec(p.exec_gate);
    io.pod(p.info);
}

}  // namespace
}  // namespace gs

using namespace gs;

extern "C" {

gs_status gs_program_save(const gs_program* prog, const char* path) {
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

gs_status gs_program_load(const char* path, gs_program** out) {
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
    // structural consistency, then the program hash over the loaded descriptors
    const Program& q = *p;
    const bool sane = q.level_off.size() == (size_t)q.n_levels + 1 && q.aux.size() == q.n_eval &&
                      q.in_lo.size() == (size_t)q.n_eval * 4 && q.term_off.size() == (size_t)q.n_eval + 1 &&
                      q.po_rows.size() == q.n_po && q.reg_init.size() == q.n_reg &&
                      q.latch_src.size() == q.latch_dst.size() && q.gate_level.size() == q.n_gates &&
                      q.coeff_off.size() == (size_t)q.n_gates + 1 && q.exec_gate.size() == q.n_eval &&
                      (!q.any_wide || q.in_hi.size() == (size_t)q.n_eval * 4) && q.hot.size() == q.n_eval &&
                      (q.level_off.empty() || q.level_off.back() == q.n_eval);
    if (!sane || program_hash(q) != q.info.program_hash)
        return fail(GS_ERR_ARG, std::string("gs_program_load: inconsistent program (hash mismatch): ") + path);
    *out = new gs_program{p.release()};
    clear_error();
    return GS_OK;
}

}  // extern "C"
