#!/usr/bin/env python
"""Kernel T vs kernel A on mid-size synthetic sequential circuits (the paper's Table I scale,
7k-372k gates): stimulus*gate*cycle/s at 65,536 lanes.  usage: python scripts/mid_size.py"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    lanes, cycles = 65536, 50
    for G, D in ((5000, 24), (10000, 28), (20000, 32), (40000, 36)):
        nl = workloads.synthetic(G, G // 25, 64, 64, D, seed=G, name=f"s{G}")
        prog = gs.Netlist.from_arrays(nl).compile()
        for kernel, flags in (("lut", 0), ("tile", 0), ("tile", 16), ("tile", 32)):
            try:
                sim = gs.Sim(prog, lanes, kernel=kernel, flags=flags)
            except gs.GsError as e:
                print(json.dumps({"gates": G, "kernel": kernel, "flags": flags, "error": str(e)}), flush=True)
                continue
            sim.bind_generated(1)
            sim.step(cycles)
            sim.sync()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sim.stream)
            sim.step(cycles * 2)
            e1.record(sim.stream)
            torch.cuda.synchronize()
            s = e0.elapsed_time(e1) / 1e3
            print(json.dumps({"gates": G, "levels": prog.info["n_levels"], "slots": prog.tile_slots(),
                              "kernel": kernel, "flags": flags, "sgc_per_s": G * lanes * cycles * 2 / s}), flush=True)
            sim.close()


if __name__ == "__main__":
    main()
