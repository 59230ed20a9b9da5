// internal.h — host-side data structures of the gsim library (not part of the ABI).
//
// See DESIGN.md §"HBM layout" for the row map and descriptor formats.
#pragma once

#include <cstdint>
#include <exception>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../include/gsim.h"

namespace gs {

// NVTX range for the duration of a C-ABI call (visible in nsys / ncu --nvtx timelines)
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};

// ---------------------------------------------------------------- errors
void set_error(const std::string& msg);
void clear_error();
gs_status fail(gs_status code, const std::string& msg);

// Every extern "C" body runs inside GS_TRY: no C++ exception crosses the ABI (gsim.h).
// Variadic, so a body with top-level commas (declarations, templates) passes through intact.
#define GS_TRY(...)                                                   \
    try {                                                             \
        __VA_ARGS__                                                   \
    } catch (const std::bad_alloc&) {                                 \
        return ::gs::fail(GS_ERR_NOMEM, "out of host memory");        \
    } catch (const std::exception& e) {                               \
        return ::gs::fail(GS_ERR_ARG, e.what());                      \
    } catch (...) {                                                   \
        return ::gs::fail(GS_ERR_ARG, "unexpected exception");        \
    }

// ---------------------------------------------------------------- netlist
enum NetKind : uint8_t { NET_PI = 0, NET_REG = 1, NET_GATE = 2 };

struct Netlist {
    std::vector<uint8_t> net_kind;      // per net
    std::vector<uint32_t> net_index;    // index within its kind
    std::vector<uint32_t> pi_net;       // net id of PI p
    std::vector<uint32_t> reg_net;      // net id of register r (its Q)
    std::vector<uint8_t> reg_init;
    std::vector<uint32_t> reg_d;        // net id, UINT32_MAX = unset
    std::vector<uint32_t> gate_net;
    std::vector<uint8_t> gate_k;
    std::vector<uint32_t> gate_in_off{0};
    std::vector<uint32_t> gate_in;      // net ids
    std::vector<uint64_t> gate_tt;
    std::vector<uint64_t> gate_tt_hi;   // [n_gates * 3] table bits 64..255, empty if no k > 6
    std::vector<uint32_t> po_net;
    uint32_t n_nets() const { return (uint32_t)net_kind.size(); }
    // the 4-word table of gate g (bits beyond 2^k are zero)
    void table(uint32_t g, uint64_t* t4) const {
        t4[0] = gate_tt[g];
        for (int j = 0; j < 3; ++j) t4[1 + j] = gate_tt_hi.empty() ? 0 : gate_tt_hi[(size_t)g * 3 + j];
    }
};

// ---------------------------------------------------------------- program
constexpr uint32_t QFLAG = 0x80000000u;   // row ref is a Q row: add the current bank offset
constexpr uint32_t GS_MAX_K_LUT64 = 6;    // widest LUT whose table fits GateAux::tt (64 bits)
constexpr uint32_t NONE32 = 0xFFFFFFFFu;

// 16-byte per-gate auxiliary descriptor (device layout, see kernels.cu)
struct GateAux {
    uint64_t tt;      // LSB-first truth table
    uint32_t qdst;    // bank-0 row of the register this gate's output also latches into, or NONE32
    uint32_t k;       // fan-in
};
static_assert(sizeof(GateAux) == 16, "GateAux layout");

struct Program {
    uint32_t n_pi = 0, n_reg = 0, n_po = 0, n_gates = 0, n_eval = 0, n_levels = 0;
    uint32_t row_pi0 = 2, row_q0 = 0, row_gate0 = 0;
    uint64_t n_rows = 0;
    bool any_wide = false;                    // some gate has k > 4
    uint32_t max_k = 0;                       // widest evaluated gate

    // execution order = level by level, k-grouped within a level
    std::vector<uint32_t> level_off;          // [n_levels + 1] into exec order
    std::vector<uint32_t> in_lo;              // [n_eval * 4] row refs (QFLAG for Q rows)
    std::vector<uint32_t> in_hi;              // [n_eval * 4] (inputs 4..7) if any_wide
    std::vector<GateAux> aux;                 // [n_eval]
    std::vector<uint64_t> tt_full;            // [n_eval * 4] 256-bit tables if max_k > 6
    std::vector<uint32_t> term_off;           // [n_eval + 1] kernel B nonzero terms
    std::vector<uint32_t> terms;              // S | (|S|-1)<<8 | (w & 0xffff)<<16
    std::vector<uint32_t> po_rows;            // [n_po]  row refs
    std::vector<uint32_t> latch_src;          // row refs
    std::vector<uint32_t> latch_dst;          // register index r
    std::vector<uint8_t> reg_init;

    // queries
    std::vector<uint32_t> gate_level;         // per netlist gate (0 for constants)
    std::vector<uint32_t> coeff_off;          // per netlist gate into coeffs
    std::vector<int32_t> coeffs;
    std::vector<uint8_t> lut_k;               // evaluated LUT of every netlist gate (after
    std::vector<uint32_t> lut_in_off, lut_in; //   optional cone collapsing): k, inputs (net
    std::vector<uint64_t> lut_tt;             //   ids) and truth table
    std::vector<uint64_t> lut_tt_hi;          //   (bits 64..255, empty if no k > 6)
    std::vector<uint32_t> exec_gate;          // exec index -> netlist gate (for G count / debug)
    gs_program_info info{};
};

gs_status compile(const Netlist& nl, const gs_compile_opts& opts, Program*& out);
uint64_t program_hash(const Program& p);

// Cone collapsing into LUTs of <= L inputs (collapse.cpp; the paper's LUT mapping)
gs_status collapse_luts(const Netlist& nl, uint32_t L, Netlist& out);

// ---------------------------------------------------------------- kernel T plan
// Shared-memory slots of one lane tile (tile.cpp): [const0, const1 | PI | Q bank 0 |
// Q bank 1 | gate values, reused by live range].
struct TileDesc {
    uint32_t in01, in23;      // input slots (16 bits each; Q refs name the bank-0 slot)
    uint32_t tt;              // truth table bits 15..0 | output slot << 16
    uint32_t kreg;            // k | (fused-latch register index + 1) << 4
};
static_assert(sizeof(TileDesc) == 16, "TileDesc layout");

struct TilePlan {
    uint32_t n_slots = 0, q0 = 0;
    std::vector<TileDesc> desc;         // [n_eval] exec order
    // narrow 8-byte descriptors {in0 | in1 << 16, tt[15:0] | out << 16}, built when every gate
    // has k <= 2, the program has no registers and no gate has k > 4 (C1, C2: half the
    // descriptor bytes, so the table fits L1 or shared memory next to more slots)
    std::vector<uint32_t> desc_n;       // [n_eval][2]
    std::vector<uint32_t> desc_hi;      // [n_eval][12] if any k > 4: in4|in5<<16, in6|in7<<16, 0, 0,
                                        //   then the 256-bit table as 8 words
    std::vector<uint32_t> po_slot;      // [n_po]
    std::vector<uint32_t> latch_src;    // slots (leftover latches)
    std::vector<uint32_t> latch_dst;    // register index
    std::vector<uint32_t> wb_row, wb_slot;   // PO values written back to state rows
};

gs_status tile_plan(const Program& p, TilePlan& t);

// Möbius transform of one LSB-first truth table of up to 2^8 bits (4 words; Algorithm 1
// as an iterative butterfly)
void mobius_butterfly(const uint64_t* tt4, uint32_t k, int32_t* w);

}  // namespace gs

struct gs_program {
    gs::Program* p;
};
