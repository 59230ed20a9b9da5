#!/usr/bin/env python
"""Fig. 6 analogue: single-stimulus-word latency
of one clock cycle against network depth over an L sweep.

The paper's Fig. 6 (UART, one stimulus) shows GPU time following the number of layers and
CPU time following the number of connections.  Here: for each circuit and L (cone
collapsing into <= L-input LUTs, lut_k), one 64-lane word (kernel A) and one 128-lane tile
(kernel T) are stepped for many cycles; the JSON lines give levels, LUTs, connections
(LUT inputs and nonzero polynomial coefficients) and microseconds per cycle,
and a summary line gives the Pearson correlation of time with levels and with connections.

usage: python scripts/fig6.py [--cycles 2000]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cycles", type=int, default=2000)
    a = ap.parse_args()
    import torch
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    circuits = {"mult32": workloads.array_multiplier(32), "adder8": workloads.adder(8),
                "synth20k": workloads.synthetic(20000, 800, 32, 48, 24, seed=12, name="s20k")}
    rows = []
    for name, nl in circuits.items():
        for L in (0, 2, 3, 4, 5, 6, 7, 8):
            prog = gs.Netlist.from_arrays(nl).compile(lut_k=L)
            info = prog.info
            for kernel, lanes in (("lut", 64), ("tile", 128)):
                try:
                    sim = gs.Sim(prog, lanes, kernel=kernel)
                except gs.GsError:
                    continue
                sim.bind_generated(1)
                sim.step(50)
                sim.sync()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(sim.stream)
                sim.step(a.cycles)
                e1.record(sim.stream)
                torch.cuda.synchronize()
                us = e0.elapsed_time(e1) * 1e3 / a.cycles
                row = {"circuit": name, "L": L, "kernel": kernel, "lanes": lanes, "levels": info["n_levels"],
                       "luts": info["n_eval_gates"], "lut_inputs": info["n_edges"],
                       "connections_nnz": info["nnz_coeffs"], "us_per_cycle": us}
                rows.append(row)
                print(json.dumps(row), flush=True)
                sim.close()
    for name in circuits:
        for kernel in ("lut", "tile"):
            r = [x for x in rows if x["circuit"] == name and x["kernel"] == kernel]
            if len(r) < 3:
                continue
            t = np.array([x["us_per_cycle"] for x in r])
            lv = np.array([x["levels"] for x in r], dtype=float)
            cn = np.array([x["connections_nnz"] for x in r], dtype=float)
            print(json.dumps({"summary": name, "kernel": kernel,
                              "pearson_time_levels": float(np.corrcoef(t, lv)[0, 1]),
                              "pearson_time_connections": float(np.corrcoef(t, cn)[0, 1])}), flush=True)


if __name__ == "__main__":
    main()
