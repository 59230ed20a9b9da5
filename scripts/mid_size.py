#!/usr/bin/env python
"""Kernel T vs kernel A on mid-size synthetic sequential circuits (the paper's Table I scale,
7k-372k gates): stimulus*gate*cycle/s.
usage: python scripts/mid_size.py [--lanes N] [--gates 5000,10000,...] [--flags 0,16,32,256]
(flags 256 = kernel T with global-memory slots)"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, default=65536)
    ap.add_argument("--gates", default="5000,10000,20000,40000")
    ap.add_argument("--flags", default="0,16,32")
    ap.add_argument("--tile-words", type=int, default=0)
    ap.add_argument("--tile-groups", type=int, default=0)
    args = ap.parse_args()
    lanes, cycles = args.lanes, 50
    depth = {5000: 24, 10000: 28, 20000: 32, 40000: 36, 100000: 40, 200000: 44, 400000: 48}
    for G in (int(x) for x in args.gates.split(",")):
        D = depth.get(G, 40)
        nl = workloads.synthetic(G, G // 25, 64, 64, D, seed=G, name=f"s{G}")
        prog = gs.Netlist.from_arrays(nl).compile()
        try:
            slots = prog.tile_slots()
        except gs.GsError:
            slots = None
        for kernel, flags in [("lut", 0)] + [("tile", int(f)) for f in args.flags.split(",")]:
            try:
                sim = gs.Sim(prog, lanes, kernel=kernel, flags=flags,
                             tile_words=args.tile_words if kernel == "tile" else 0,
                             tile_groups=args.tile_groups if kernel == "tile" else 0)
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
            print(json.dumps({"gates": G, "lanes": lanes, "levels": prog.info["n_levels"], "slots": slots,
                              "kernel": kernel, "flags": flags, "sgc_per_s": G * lanes * cycles * 2 / s,
                              "launch": sim.launch}), flush=True)
            sim.close()


if __name__ == "__main__":
    main()
