"""Fig. 6 analogue, CPU half (§IV-B, caption P:332).

The paper compiles one circuit at several LUT sizes L and times a single-stimulus simulation
of the resulting network on the CPU (non-parallel) and on the GPU: CPU time follows the
number of NN connections (it is a sparse matrix product), GPU time follows the
number of layers.  The CPU side here is the ORACLE in its network mode (mode 'poly': every
gate evaluated as the two-layer network of Fig. 2 / Eq. 1-3, the dense hidden layer of all
2^k monomials), on one thread, over cone-collapsed versions of the same circuit for L = 2..8
(the LUT netlists come from gs_program_gate_lut, as in test_collapse.py, which checks that
they simulate identically).  The GPU half (latency against levels) is scripts/fig6.py.

Property checked (the paper's claim): across the L sweep, CPU time correlates with the
connection count (Pearson > 0.95).  With GS_FIG6_OUT=<file> the series and the Pearson
coefficients are written as JSON lines (profiles/r02_fig6_cpu_oracle.jsonl).
"""
import json
import os
import time

import numpy as np
import pytest

import oracle
import workloads
from tests.test_collapse import collapsed_netlist

CIRCUITS = {"adder8": lambda: workloads.adder(8), "mult32": lambda: workloads.array_multiplier(32),
            "synth20k": lambda: workloads.synthetic(20000, 800, 32, 48, 24, seed=12, name="s20k")}
LS = (0, 2, 3, 4, 5, 6, 7, 8)
BLOCK = 16          # the oracle advances lanes in 16-lane blocks: time one full block


def connection_counts(nl):
    """(dense, nnz) connections of the network the LUT netlist compiles to (Fig. 2): a k-input
    LUT has 2^k hidden neurons h_S with |S| input weights each and one output weight per
    neuron — k 2^(k-1) + 2^k dense; the sparse network keeps the neurons with w_S != 0
    (P:187), sum over them of |S| + 1.  Coefficients from the oracle's own definition."""
    dense = nnz = 0
    for g in range(nl.n_gates):
        k = int(nl.gate_k[g])
        if k == 0:
            continue
        dense += k * 2 ** (k - 1) + 2 ** k
        words = [int(nl.gate_tt[g])] + ([int(x) for x in nl.gate_tt_hi[g]] if nl.gate_tt_hi is not None else [])
        w = oracle.mobius_def_wide(words[:max(1, (1 << k) // 64)], k)
        nnz += sum(bin(S).count("1") + 1 for S in range(1 << k) if w[S] != 0)
    return dense, nnz


def cpu_time_per_cycle(nl, mode):
    lanes = np.arange(BLOCK)
    c = 2
    while True:
        t = time.perf_counter()
        oracle.simulate(nl, lanes, c, seed=1, mode=mode, threads=1, want=("sig",))
        dt = time.perf_counter() - t
        if dt > 0.15 or c >= 4096:
            return dt / c
        c *= 4


@pytest.mark.parametrize("name", list(CIRCUITS))
def test_cpu_network_time_follows_connections(name):
    nl = CIRCUITS[name]()
    rows = []
    for L in LS:
        c = nl if L == 0 else collapsed_netlist(nl, L)[1]
        dense, nnz = connection_counts(c)
        levels = int(oracle.asap_levels(c).max())
        t_poly = cpu_time_per_cycle(c, "poly")
        rows.append({"circuit": name, "L": L, "luts": int((c.gate_k > 0).sum()), "levels": levels,
                     "connections_dense": dense, "connections_nnz": nnz,
                     "oracle_poly_us_per_cycle_16_lanes": t_poly * 1e6, "threads": 1})
    t = np.array([r["oracle_poly_us_per_cycle_16_lanes"] for r in rows])
    dn = np.array([r["connections_dense"] for r in rows], dtype=float)
    nz = np.array([r["connections_nnz"] for r in rows], dtype=float)
    lv = np.array([r["levels"] for r in rows], dtype=float)
    summary = {"summary": name, "pearson_cpu_time_connections_dense": float(np.corrcoef(t, dn)[0, 1]),
               "pearson_cpu_time_connections_nnz": float(np.corrcoef(t, nz)[0, 1]),
               "pearson_cpu_time_levels": float(np.corrcoef(t, lv)[0, 1])}
    out = os.environ.get("GS_FIG6_OUT")
    if out:
        with open(out, "a") as f:
            for r in rows + [summary]:
                f.write(json.dumps(r) + "\n")
    assert summary["pearson_cpu_time_connections_dense"] > 0.95, summary
