/*
 * oracle/oracle.c — CPU ORACLE. TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this code.  It shares no code, header, table or
 * constant generator with the CUDA path (paper_conf_ipps_gavierrprs23_b200/);
 * neither side includes or imports the other.
 *
 * What it computes (DESIGN.md §"Oracle"): the plain cycle-based simulation of
 * a digital circuit f:{0,1}^n -> {0,1}^m with D flip-flops cut into
 * pseudo-inputs / pseudo-outputs and a recurrent connection (PAPER.md P:122,
 * §II-B; §III-C "Flip-flop cuts"), one stimulus (lane) at a time,
 * one gate at a time, in a topological order of the gate DAG (§III-B1).
 * The paper's claim is exact equivalence, so the oracle is the
 * plain definition: no bit-packing, no levels, no blocking, no fusion.
 *
 * Two per-gate evaluators, selectable per call:
 *   mode 0 (TT)   v = bit idx of the truth table, idx = sum_i x_i 2^i
 *                 (the LUT of P:165 Fig. 3, LSB-first reading R1);
 *   mode 1 (POLY) v = sum_S w_S h_S  (Eq. 1) with hidden neurons
 *                 h_S = Theta(sum_{s in S} x_s - |S| + 1)  (Eq. 3),
 *                 Theta(x) = 1 iff x > 0 (Eq. 2), and w_S computed by
 *                 the inclusion-exclusion definition of the multilinear
 *                 coefficients (orc_mobius_def).  A result outside {0,1}
 *                 (impossible by P:224) is counted as an invariant violation.
 *
 * Stimulus, register-init, output-sampling, MISR and lane-signature rules are
 * DESIGN.md readings R2-R6; every helper below restates one.
 *
 * Pins (tests/test_oracle_*.py): splitmix64 / CRC-64-ECMA published values,
 * adder = a+b exhaustively, multiplier = a*b, LFSR16 period 65535 and sequence,
 * counters mod 2^n, register delay lines / hold / swap closed forms, brute force
 * against a recursive evaluator on tiny netlists, polynomial == truth table on
 * all 65,536 4-input functions, textbook Möbius closed forms.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---------------------------------------------------------------- hashing */

/* splitmix64 finaliser with the golden-gamma increment (reading R2). */
uint64_t orc_mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* PI word hash H(seed, p, c, w) = mix64(mix64(mix64(seed ^ p) ^ c) ^ w); lane s
 * reads bit (s mod 64) of H(seed, p, c, floor(s / 64))  (reading R2). */
uint64_t orc_stim_word(uint64_t seed, uint64_t p, uint64_t c, uint64_t w) {
    return orc_mix64(orc_mix64(orc_mix64(seed ^ p) ^ c) ^ w);
}

/* One MISR clock: sig' = (sig << 1) ^ (msb ? CRC-64/ECMA-182 poly : 0) ^ v (R5). */
uint64_t orc_misr_step(uint64_t sig, uint64_t v) {
    uint64_t fb = (sig >> 63) ? 0x42F0E1EBA9EA3693ULL : 0ULL;
    return (sig << 1) ^ fb ^ v;
}

/* Per-lane term of the job signature: mix64(sig_s ^ mix64(s)) (R6). */
uint64_t orc_lane_sig_term(uint64_t sig, uint64_t s) {
    return orc_mix64(sig ^ orc_mix64(s));
}

/* ------------------------------------------------- multilinear polynomial */

static int popc(uint32_t x) { int n = 0; while (x) { n += x & 1u; x >>= 1; } return n; }

/* Coefficients of the unique multilinear polynomial of a k-input function
 * (Eq. 1), by their definition:  w_S = sum_{T subset S} (-1)^{|S|-|T|} f(1_T).
 * Index bit i of S <-> variable x_i is in S (LSB-first, reading R1). */
void orc_mobius_def(uint64_t tt, int k, int64_t* w) {
    uint32_t n = 1u << k;
    for (uint32_t S = 0; S < n; ++S) {
        int64_t acc = 0;
        for (uint32_t T = 0; T < n; ++T) {
            if ((T & ~S) != 0) continue;                 /* T must be a subset of S */
            int64_t f = (int64_t)((tt >> T) & 1u);
            acc += ((popc(S) - popc(T)) & 1) ? -f : f;
        }
        w[S] = acc;
    }
}

/* The same definition for tables of up to 2^8 entries given as 4 uint64 words (k <= 8). */
void orc_mobius_def_wide(const uint64_t* tt4, int k, int64_t* w) {
    uint32_t n = 1u << k;
    for (uint32_t S = 0; S < n; ++S) {
        int64_t acc = 0;
        for (uint32_t T = 0; T < n; ++T) {
            if ((T & ~S) != 0) continue;                 /* T must be a subset of S */
            int64_t f = (int64_t)((tt4[T >> 6] >> (T & 63)) & 1u);
            acc += ((popc(S) - popc(T)) & 1) ? -f : f;
        }
        w[S] = acc;
    }
}

/* The two-layer network of Fig. 2 for one input point x (bit i = x_i):
 * hidden neuron h_S = Theta(sum_{s in S} x_s - |S| + 1) (Eq. 3, weights 1,
 * bias |S|-1), Theta(z) = [z > 0] (Eq. 2); output = sum_S w_S h_S (Eq. 1),
 * no bias, no threshold. */
int64_t orc_poly_eval(const int64_t* w, int k, uint32_t x) {
    int64_t out = 0;
    for (uint32_t S = 0; S < (1u << k); ++S) {
        int64_t z = 0;
        for (int s = 0; s < k; ++s)
            if ((S >> s) & 1u) z += (x >> s) & 1u;
        z = z - popc(S) + 1;
        int64_t h = z > 0 ? 1 : 0;
        out += w[S] * h;
    }
    return out;
}

/* ------------------------------------------------------------ the netlist */

/* Netlist arrays (format documented in workloads/netlists.py; the oracle has
 * its own reader — nothing here is shared with the library). */
typedef struct {
    uint32_t n_pi, n_reg, n_gates, n_po;
    const uint8_t*  reg_init;
    const uint32_t* reg_d;
    const uint8_t*  gate_k;
    const uint32_t* gate_in_off;
    const uint32_t* gate_in;
    const uint64_t* gate_tt;
    const uint32_t* po;
    const uint64_t* gate_tt_hi;   /* [n_gates][3]: table bits 64..255 (k = 7, 8), or NULL */
} orc_netlist;

/* Bit idx of gate g's truth table (LSB-first, reading R1); tables of k = 7, 8 gates continue
 * into gate_tt_hi. */
static uint32_t tt_bit(const orc_netlist* nl, uint32_t g, uint32_t idx) {
    if (idx < 64) return (uint32_t)((nl->gate_tt[g] >> idx) & 1u);
    return (uint32_t)((nl->gate_tt_hi[(uint64_t)g * 3 + (idx >> 6) - 1] >> (idx & 63)) & 1u);
}

/* binary min-heap of gate ids (for the topological order below) */
static void heap_push(uint32_t* h, uint32_t* n, uint32_t v) {
    uint32_t i = (*n)++;
    while (i > 0) {
        uint32_t p = (i - 1) / 2;
        if (h[p] <= v) break;
        h[i] = h[p];
        i = p;
    }
    h[i] = v;
}
static uint32_t heap_pop(uint32_t* h, uint32_t* n) {
    uint32_t top = h[0], v = h[--(*n)], i = 0;
    for (;;) {
        uint32_t c = 2 * i + 1;
        if (c >= *n) break;
        if (c + 1 < *n && h[c + 1] < h[c]) c++;
        if (v <= h[c]) break;
        h[i] = h[c];
        i = c;
    }
    if (*n) h[i] = v;
    return top;
}

/* Kahn topological order of the gate DAG: a gate is ready when all of
 * its gate inputs are done; among ready gates the smallest id goes first.
 * Returns 0, or -1 on a combinational loop (reading R8) or a bad net id. */
int orc_topo_order(const orc_netlist* nl, uint32_t* order) {
    uint32_t G = nl->n_gates, base = nl->n_pi + nl->n_reg;
    uint32_t* indeg = (uint32_t*)calloc(G ? G : 1, sizeof(uint32_t));
    uint32_t* cnt = (uint32_t*)calloc(G + 1, sizeof(uint32_t));
    uint32_t E = nl->gate_in_off[G];
    uint32_t* adj = (uint32_t*)malloc((E ? E : 1) * sizeof(uint32_t));
    int rc = 0;
    for (uint32_t g = 0; g < G; ++g)
        for (uint32_t e = nl->gate_in_off[g]; e < nl->gate_in_off[g + 1]; ++e) {
            uint32_t n = nl->gate_in[e];
            if (n >= base + G) { rc = -1; goto done; }
            if (n >= base) { indeg[g]++; cnt[n - base + 1]++; }
        }
    for (uint32_t g = 0; g < G; ++g) cnt[g + 1] += cnt[g];
    {
        uint32_t* fill = (uint32_t*)calloc(G ? G : 1, sizeof(uint32_t));
        for (uint32_t g = 0; g < G; ++g)
            for (uint32_t e = nl->gate_in_off[g]; e < nl->gate_in_off[g + 1]; ++e) {
                uint32_t n = nl->gate_in[e];
                if (n >= base) { uint32_t p = n - base; adj[cnt[p] + fill[p]++] = g; }
            }
        free(fill);
    }
    {
        /* Kahn's algorithm taking the ready gate with the SMALLEST id first (a binary
         * min-heap): the lexicographically first topological order, which is plain id
         * order whenever every gate's inputs have smaller ids (SURVEY §8(c) "Kahn, by gate
         * id").  Any topological order gives the same values (reading R11). */
        uint32_t* heap = (uint32_t*)malloc((G ? G : 1) * sizeof(uint32_t));
        uint32_t hn = 0, tail = 0;
        for (uint32_t g = 0; g < G; ++g) if (indeg[g] == 0) heap_push(heap, &hn, g);
        while (hn) {
            uint32_t g = heap_pop(heap, &hn);
            order[tail++] = g;
            for (uint32_t e = cnt[g]; e < cnt[g + 1]; ++e)
                if (--indeg[adj[e]] == 0) heap_push(heap, &hn, adj[e]);
        }
        free(heap);
        if (tail != G) rc = -1;
    }
done:
    free(indeg); free(cnt); free(adj);
    return rc;
}

/* Longest-path depth of every gate: level(g) = 1 + max(level(inputs)), PIs, Qs
 * and k=0 constants at 0 — the number of merged NN layers.  */
int orc_asap_levels(const orc_netlist* nl, uint32_t* level) {
    uint32_t G = nl->n_gates, base = nl->n_pi + nl->n_reg;
    uint32_t* order = (uint32_t*)malloc((G ? G : 1) * sizeof(uint32_t));
    if (orc_topo_order(nl, order) != 0) { free(order); return -1; }
    for (uint32_t i = 0; i < G; ++i) {
        uint32_t g = order[i], l = 0;
        if (nl->gate_k[g] == 0) { level[g] = 0; continue; }
        for (uint32_t e = nl->gate_in_off[g]; e < nl->gate_in_off[g + 1]; ++e) {
            uint32_t n = nl->gate_in[e];
            uint32_t ln = n >= base ? level[n - base] : 0;
            if (ln > l) l = ln;
        }
        level[g] = l + 1;
    }
    free(order);
    return 0;
}

/* ------------------------------------------------------------- simulation */

#define ORC_BLOCK_MAX 64   /* most lanes a thread advances in lockstep (see orc_simulate) */

/* Lanes [0, nlanes) in blocks of B lane slots; slots past the last lane repeat the block's
 * first lane and are never reported (a fixed trip count keeps the lane loops simple).
 * Inlined with a literal B by orc_simulate. */
static inline __attribute__((always_inline)) int64_t sim_blocks(
        const orc_netlist* nl, int mode, uint64_t seed, const uint64_t* host_stim, uint64_t stim_words,
        uint32_t cycles, const uint64_t* lanes, uint32_t nlanes, const uint32_t* order,
        const uint32_t* woff, const int64_t* wall, uint8_t* trace, uint8_t* last, uint8_t* regs,
        uint64_t* sig, const uint32_t B) {
    uint32_t G = nl->n_gates, P = nl->n_pi, R = nl->n_reg, O = nl->n_po;
    uint32_t base = P + R, N = base + G;
    int64_t violations = 0;
    const int64_t nblocks = ((int64_t)nlanes + B - 1) / B;
#ifdef _OPENMP
#pragma omp parallel reduction(+ : violations)
#endif
    {
        uint8_t* v = (uint8_t*)malloc((size_t)(N ? N : 1) * B);     /* v[net * B + b] */
        uint8_t* q = (uint8_t*)malloc((size_t)(R ? R : 1) * B);     /* Q(c)   [r * B + b] */
        uint8_t* qn = (uint8_t*)malloc((size_t)(R ? R : 1) * B);    /* Q(c+1) */
        uint64_t misr[ORC_BLOCK_MAX];
        uint64_t lane[ORC_BLOCK_MAX];
#ifdef _OPENMP
#pragma omp for schedule(dynamic, 1)
#endif
        for (int64_t bi = 0; bi < nblocks; ++bi) {
            const uint64_t l0 = (uint64_t)bi * B;
            const uint32_t nb = (uint32_t)((l0 + B <= nlanes) ? B : nlanes - l0);
            for (uint32_t b = 0; b < B; ++b) {
                lane[b] = lanes[l0 + (b < nb ? b : 0)];
                misr[b] = 0;
            }
            for (uint32_t r = 0; r < R; ++r)
                for (uint32_t b = 0; b < B; ++b) q[(size_t)r * B + b] = nl->reg_init[r] & 1u;
            for (uint32_t c = 0; c < cycles; ++c) {
                for (uint32_t p = 0; p < P; ++p)
                    for (uint32_t b = 0; b < B; ++b) {
                        const uint64_t s = lane[b];
                        uint64_t word = host_stim ? host_stim[((uint64_t)c * P + p) * stim_words + (s >> 6)]
                                                  : orc_stim_word(seed, p, c, s >> 6);
                        v[(size_t)p * B + b] = (uint8_t)((word >> (s & 63)) & 1u);
                    }
                memcpy(v + (size_t)P * B, q, (size_t)R * B);
                for (uint32_t i = 0; i < G; ++i) {
                    const uint32_t g = order[i];
                    const uint32_t k = nl->gate_k[g];
                    const uint32_t* in = nl->gate_in + nl->gate_in_off[g];
                    uint8_t idx[ORC_BLOCK_MAX];               /* truth-table index of every lane (R1), k <= 8 */
                    for (uint32_t b = 0; b < B; ++b) idx[b] = 0;
                    for (uint32_t j = 0; j < k; ++j) {
                        const uint8_t* restrict x = v + (size_t)in[j] * B;
                        for (uint32_t b = 0; b < B; ++b) idx[b] |= (uint8_t)(x[b] << j);
                    }
                    uint8_t* restrict y = v + (size_t)(base + g) * B;
                    if (mode == 1) {
                        for (uint32_t b = 0; b < B; ++b) {
                            int64_t val = orc_poly_eval(wall + woff[g], (int)k, idx[b]);
                            if (b < nb && val != 0 && val != 1) violations++;
                            y[b] = (uint8_t)(val & 1);
                        }
                    } else if (k <= 6) {
                        const uint64_t tt = nl->gate_tt[g];
                        for (uint32_t b = 0; b < B; ++b) y[b] = (uint8_t)((tt >> idx[b]) & 1u);
                    } else {
                        for (uint32_t b = 0; b < B; ++b) y[b] = (uint8_t)tt_bit(nl, g, idx[b]);
                    }
                }
                for (uint32_t b = 0; b < nb; ++b) {
                    const uint64_t li = l0 + b;
                    uint64_t word = 0;
                    for (uint32_t o = 0; o < O; ++o) {
                        uint8_t x = v[(size_t)nl->po[o] * B + b];
                        if (trace) trace[((uint64_t)li * cycles + c) * O + o] = x;
                        if (last && c + 1 == cycles) last[(uint64_t)li * O + o] = x;
                        word ^= (uint64_t)x << (o & 63);
                    }
                    misr[b] = orc_misr_step(misr[b], word);
                }
                for (uint32_t r = 0; r < R; ++r)
                    memcpy(qn + (size_t)r * B, v + (size_t)nl->reg_d[r] * B, B);
                memcpy(q, qn, (size_t)R * B);
            }
            for (uint32_t b = 0; b < nb; ++b) {
                const uint64_t li = l0 + b;
                if (regs)
                    for (uint32_t r = 0; r < R; ++r) regs[li * R + r] = q[(size_t)r * B + b];
                if (sig) sig[li] = misr[b];
            }
        }
        free(v); free(q); free(qn);
    }
    return violations;
}

/*
 * Simulate `nlanes` lanes (global stimulus indices lanes[i]) for `cycles`
 * clock cycles.  For lane s and cycle c:
 *   PI_p(c,s) = bit (s mod 64) of stim word:  host_stim == NULL ->
 *               orc_stim_word(seed, p, c, s/64);  else
 *               host_stim[(c * n_pi + p) * stim_words + s/64]   ("binary inputs")
 *   Q_r(0,s)  = reg_init[r]                                     (reading R3)
 *   gates in topological order, TT lookup (mode 0) or Eq. 1-3 network (mode 1)
 *   out_o(c,s)= value of net po[o] after the evaluation, before the latch (R4)
 *   Q_r(c+1,s)= value of net reg_d[r] in cycle c, all registers at once (R3)
 *   sig_s     = orc_misr_step(sig_s, xor_o out_o(c,s) << (o mod 64))  (R5)
 * Lanes never interact (stimulus independence), so a thread advances a block of up
 * to ORC_BLOCK_MAX lanes in lockstep: per cycle it visits every gate once in the topological
 * order and applies the same per-lane rule to each lane of the block (one byte per lane
 * and net; no bit packing).  The netlist tables are then read once per block and cycle
 * instead of once per lane and cycle; the value of every lane is computed exactly as in
 * the one-lane formulation above.
 * Outputs (any may be NULL):
 *   trace  [nlanes][cycles][n_po] bytes  — every output of every cycle
 *   last   [nlanes][n_po] bytes          — outputs of the last cycle
 *   regs   [nlanes][n_reg] bytes         — Q after the last clock edge, Q(cycles)
 *   sig    [nlanes] uint64               — per-lane MISR
 * Returns the number of polynomial invariant violations (mode 1), or -1 on error.
 */
int64_t orc_simulate(const orc_netlist* nl, int mode, uint64_t seed,
                     const uint64_t* host_stim, uint64_t stim_words,
                     uint32_t cycles, const uint64_t* lanes, uint32_t nlanes, int threads,
                     uint8_t* trace, uint8_t* last, uint8_t* regs, uint64_t* sig) {
    uint32_t G = nl->n_gates, P = nl->n_pi, R = nl->n_reg, O = nl->n_po;
    uint32_t base = P + R, N = base + G;
    uint32_t* order = (uint32_t*)malloc((G ? G : 1) * sizeof(uint32_t));
    if (orc_topo_order(nl, order) != 0) { free(order); return -1; }
    for (uint32_t r = 0; r < R; ++r) if (nl->reg_d[r] >= N) { free(order); return -1; }
    for (uint32_t g = 0; g < G; ++g)
        if (nl->gate_k[g] > 8 || (nl->gate_k[g] > 6 && !nl->gate_tt_hi)) { free(order); return -1; }
    for (uint32_t o = 0; o < O; ++o) if (nl->po[o] >= N) { free(order); return -1; }

    /* coefficients of every gate, by definition (mode 1 only) */
    uint32_t* woff = NULL;
    int64_t* wall = NULL;
    if (mode == 1) {
        woff = (uint32_t*)malloc((G + 1) * sizeof(uint32_t));
        woff[0] = 0;
        for (uint32_t g = 0; g < G; ++g) woff[g + 1] = woff[g] + (1u << nl->gate_k[g]);
        wall = (int64_t*)malloc((woff[G] ? woff[G] : 1) * sizeof(int64_t));
        for (uint32_t g = 0; g < G; ++g) {
            uint64_t tt4[4] = {nl->gate_tt[g], 0, 0, 0};
            if (nl->gate_k[g] > 6)
                for (int j = 0; j < 3; ++j) tt4[1 + j] = nl->gate_tt_hi[(uint64_t)g * 3 + j];
            orc_mobius_def_wide(tt4, nl->gate_k[g], wall + woff[g]);
        }
    }

#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
#endif
    /* lanes per block: 64 (one cache line per net and block) when there are enough lanes
     * for every thread, else 32 or 16 */
    uint32_t nth = 1;
#ifdef _OPENMP
    nth = (uint32_t)omp_get_max_threads();
#endif
    int64_t violations;
    if ((uint64_t)nlanes >= 64ull * nth)
        violations = sim_blocks(nl, mode, seed, host_stim, stim_words, cycles, lanes, nlanes, order, woff, wall,
                                trace, last, regs, sig, 64);
    else if ((uint64_t)nlanes >= 32ull * nth)
        violations = sim_blocks(nl, mode, seed, host_stim, stim_words, cycles, lanes, nlanes, order, woff, wall,
                                trace, last, regs, sig, 32);
    else
        violations = sim_blocks(nl, mode, seed, host_stim, stim_words, cycles, lanes, nlanes, order, woff, wall,
                                trace, last, regs, sig, 16);
    free(order); free(woff); free(wall);
    return violations;
}

int orc_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
