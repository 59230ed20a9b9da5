/*
 * examples/adder_c_abi.c — the C-ABI used from plain C (no Python, no torch): build an 8-bit
 * ripple-carry adder gate by gate (gs_add_*), compile it (levels + Möbius coefficients),
 * simulate all 65,536 input pairs in one batch (64 stimuli per word), read the outputs back
 * and check sum = a + b.  Device memory comes from cudaMalloc (caller-owned workspace).
 *
 *   gcc -O2 -std=c11 -Iinclude -I/usr/local/cuda/include examples/adder_c_abi.c \
 *       -Lpaper_conf_ipps_gavierrprs23_b200 -lgsim -L/usr/local/cuda/lib64 -lcudart \
 *       -Wl,-rpath,$PWD/paper_conf_ipps_gavierrprs23_b200 -o build_examples/adder_c_abi
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <cuda_runtime.h>

#include "gsim.h"

#define CHECK(call)                                                                       \
    do {                                                                                  \
        gs_status st_ = (call);                                                           \
        if (st_ != GS_OK) {                                                               \
            fprintf(stderr, "%s failed: %d %s\n", #call, (int)st_, gs_last_error());      \
            return 1;                                                                     \
        }                                                                                 \
    } while (0)

enum { XOR2 = 0x6, AND2 = 0x8, OR2 = 0xE };   /* LSB-first 2-input truth tables */

int main(void) {
    gs_netlist* nl;
    CHECK(gs_netlist_create(&nl));
    gs_net a[8], b[8], carry = 0;
    for (int i = 0; i < 8; ++i) CHECK(gs_add_input(nl, &a[i]));
    for (int i = 0; i < 8; ++i) CHECK(gs_add_input(nl, &b[i]));
    for (int i = 0; i < 8; ++i) {
        gs_net in2[2] = {a[i], b[i]}, t, s, g;
        CHECK(gs_add_gate(nl, 2, in2, XOR2, &t));
        CHECK(gs_add_gate(nl, 2, in2, AND2, &g));
        if (i == 0) {
            s = t;
            carry = g;
        } else {
            gs_net tc[2] = {t, carry}, p, gp[2];
            CHECK(gs_add_gate(nl, 2, tc, XOR2, &s));
            CHECK(gs_add_gate(nl, 2, tc, AND2, &p));
            gp[0] = g; gp[1] = p;
            CHECK(gs_add_gate(nl, 2, gp, OR2, &carry));
        }
        CHECK(gs_mark_output(nl, s, NULL));
    }
    CHECK(gs_mark_output(nl, carry, NULL));

    gs_compile_opts copts;
    memset(&copts, 0, sizeof(copts));
    copts.balance = 1;
    gs_program* prog;
    CHECK(gs_compile(nl, &copts, &prog));
    gs_program_info info;
    CHECK(gs_program_get_info(prog, &info));

    const uint64_t lanes = 1u << 16, words = lanes / 64;
    gs_sim_opts so;
    memset(&so, 0, sizeof(so));
    so.lanes = lanes;
    so.kernel = GS_KERNEL_AUTO;
    so.use_graphs = 1;
    size_t bytes;
    CHECK(gs_sim_workspace_bytes(prog, &so, &bytes));
    void* ws;
    if (cudaMalloc(&ws, bytes) != cudaSuccess) { fprintf(stderr, "cudaMalloc failed\n"); return 1; }
    gs_sim* sim;
    CHECK(gs_sim_create(prog, &so, ws, bytes, &sim));

    /* stimulus [cycle][pi][word]: lane s carries a = s & 0xff, b = s >> 8 */
    uint64_t* stim = calloc(16 * words, sizeof(uint64_t));
    for (uint64_t s = 0; s < lanes; ++s)
        for (int p = 0; p < 16; ++p)
            if ((s >> p) & 1) stim[p * words + s / 64] |= 1ull << (s % 64);
    CHECK(gs_sim_bind_stimulus_host(sim, stim, 1));
    CHECK(gs_sim_step(sim, 1));
    uint64_t* out = calloc(9 * words, sizeof(uint64_t));
    CHECK(gs_sim_read_outputs(sim, out, 9 * words));
    uint64_t bad = 0;
    for (uint64_t s = 0; s < lanes; ++s) {
        unsigned sum = 0;
        for (int o = 0; o < 9; ++o) sum |= (unsigned)((out[o * words + s / 64] >> (s % 64)) & 1) << o;
        if (sum != (s & 0xff) + (s >> 8)) ++bad;
    }
    printf("adder_c_abi: %u gates, %u levels, %llu lanes, %llu mismatches\n", info.n_eval_gates,
           info.n_levels, (unsigned long long)lanes, (unsigned long long)bad);
    CHECK(gs_sim_destroy(sim));
    CHECK(gs_program_destroy(prog));
    CHECK(gs_netlist_destroy(nl));
    cudaFree(ws);
    free(stim);
    free(out);
    return bad ? 2 : 0;
}
