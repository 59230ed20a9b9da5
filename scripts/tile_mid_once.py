#!/usr/bin/env python
"""Kernel T on a mid-size synthetic circuit in a fresh process: ~1 s of warm-up steps (the GPU
clock ramps from idle), then ~1 s of timed steps of --cycles cycles; --gates G --flags F --tw TW
--ng NG.  Also an ncu target."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

ap = argparse.ArgumentParser()
ap.add_argument("--gates", type=int, default=5000)
ap.add_argument("--flags", type=int, default=0)
ap.add_argument("--tw", type=int, default=0)
ap.add_argument("--ng", type=int, default=0)
ap.add_argument("--cycles", type=int, default=10)
a = ap.parse_args()
import workloads
import paper_conf_ipps_gavierrprs23_b200 as gs
depth = {5000: 24, 10000: 28, 20000: 32, 40000: 36}
nl = workloads.synthetic(a.gates, a.gates // 25, 64, 64, depth.get(a.gates, 40), seed=a.gates, name="m")
prog = gs.Netlist.from_arrays(nl).compile()
sim = gs.Sim(prog, 65536, kernel="tile", flags=a.flags, tile_words=a.tw, tile_groups=a.ng)
import json
import time
import torch
sim.bind_generated(1)
# warm the GPU up for ~1 s (clocks ramp from idle), then time ~1 s of steps
t = time.time()
while time.time() - t < 1.0:
    sim.step(a.cycles)
    sim.sync()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(sim.stream)
e1.record(sim.stream)
e1.synchronize()
n = 0
e0.record(sim.stream)
t = time.time()
while time.time() - t < 1.0:
    sim.step(a.cycles)
    n += 1
e1.record(sim.stream)
torch.cuda.synchronize()
s = e0.elapsed_time(e1) / 1e3
print(json.dumps({"gates": a.gates, "flags": a.flags, "sgc_per_s": a.gates * 65536 * a.cycles * n / s,
                  "steps": n, "launch": sim.launch}))
