#!/usr/bin/env python
"""The paper's L sweep (Table I L = 3/7/11, Fig. 6) on the structural and
synthetic configs: compile with cone collapsing into <= L-input LUTs and time the hot path.

Prints one JSON line per (config, L, kernel): levels, evaluated LUTs, LUT inputs, and two
throughputs — `lut_sgc_per_s` counts the evaluated LUTs (the headline metric's unit) and
`circuit_gcps` counts the ORIGINAL circuit's gates, as the paper's Table I does (P:271,
P:291), so it rises when collapsing makes the same circuit faster.

usage: python scripts/l_sweep.py [--configs C1,C2,C3] [--cycles 100] [--steps 3]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3")
    ap.add_argument("--Ls", default="0,3,4,5,6,7,8")
    ap.add_argument("--kernels", default="lut,auto,poly")
    ap.add_argument("--cycles", type=int, default=100)
    ap.add_argument("--steps", type=int, default=3)
    a = ap.parse_args()
    import torch
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    for name in a.configs.split(","):
        cfg = workloads.CONFIGS[name]
        nl = cfg.netlist()
        g_orig = int((nl.gate_k > 0).sum())
        lanes = cfg.lanes if cfg.shards == 1 else cfg.lanes // cfg.shards
        for L in (int(x) for x in a.Ls.split(",")):
            prog = gs.Netlist.from_arrays(nl).compile(lut_k=L)
            info = prog.info
            for kernel in a.kernels.split(","):
                stream = torch.cuda.Stream()
                try:
                    sim = gs.Sim(prog, lanes, kernel=kernel, stream=stream)
                except gs.GsError:               # k > 6 LUTs: kernel B only
                    continue
                sim.bind_generated(cfg.stim_seed)
                sim.step(a.cycles)
                sim.sync()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                for _ in range(a.steps):
                    sim.step(a.cycles)
                e1.record(stream)
                torch.cuda.synchronize()
                s = e0.elapsed_time(e1) / 1e3
                evals = lanes * a.cycles * a.steps
                print(json.dumps({"config": name, "L": L, "kernel": kernel,
                                  "kernel_used": ("tile" if sim.launches_per_cycle() == 1 else
                                                  "lut" if kernel == "auto" else kernel),
                                  "levels": info["n_levels"], "luts": info["n_eval_gates"],
                                  "lut_inputs": info["n_edges"], "nnz_coeffs": info["nnz_coeffs"],
                                  "gates_original": g_orig, "lanes": lanes,
                                  "ms_per_cycle": s * 1e3 / (a.cycles * a.steps),
                                  "lut_sgc_per_s": info["n_eval_gates"] * evals / s,
                                  "circuit_gcps": g_orig * evals / s}), flush=True)
                sim.close()


if __name__ == "__main__":
    main()
