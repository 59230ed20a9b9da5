"""Experiment: split one GPU's lanes into N independent sub-batches, each a gs_sim on its own
CUDA stream, so the per-level kernels of different sub-batches overlap (latency-bound
mid-size circuits: each level is only ~0.5 wave deep).  Prints one JSON line per (config,
N, kernel) with sgc/s; lane_sig_sum of the union is checked equal for every N.

usage: python scripts/split_streams.py [--configs C3] [--splits 1,2,4] [--cycles 100]
"""
import argparse
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads  # noqa: E402
import paper_conf_ipps_gavierrprs23_b200 as gs  # noqa: E402


def run(prog, lanes, n, kernel, cycles, steps, seed, flags=0):
    streams = [torch.cuda.Stream() for _ in range(n)]
    sub = lanes // n
    sims = [gs.Sim(prog, sub, lane_offset=i * sub, kernel=kernel, stream=streams[i], flags=flags)
            for i in range(n)]
    for s in sims:
        s.bind_generated(seed)
    main = torch.cuda.current_stream()

    def step():
        ev = torch.cuda.Event()
        ev.record(main)
        for st, s in zip(streams, sims):
            st.wait_event(ev)
            s.step(cycles)
        for st in streams:
            e = torch.cuda.Event()
            e.record(st)
            main.wait_event(e)

    for _ in range(2):
        step()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main)
    for _ in range(steps):
        step()
    e1.record(main)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    sig = sum(s.signature()["lane_sig_sum"] for s in sims) % (1 << 64)
    for s in sims:
        s.close()
    return ms, sig


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C3")
    ap.add_argument("--splits", default="1,2,4")
    ap.add_argument("--kernels", default="lut")
    ap.add_argument("--cycles", type=int, default=100)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--lanes", type=int, default=0)
    a = ap.parse_args()
    for cname in a.configs.split(","):
        cfg = workloads.CONFIGS[cname]
        nl = cfg.netlist()
        prog = gs.Netlist.from_arrays(nl).compile()
        G = prog.info["n_eval_gates"]
        lanes = a.lanes or cfg.lanes // getattr(cfg, "shards", 1)
        for kernel in a.kernels.split(","):
            ref = None
            for n in [int(x) for x in a.splits.split(",")]:
                ms, sig = run(prog, lanes, n, kernel, a.cycles, a.steps, cfg.stim_seed)
                ref = sig if ref is None else ref
                print(json.dumps({"config": cname, "kernel": kernel, "lanes": lanes, "split": n,
                                  "sgc_s": G * lanes * a.cycles * a.steps / (ms / 1e3),
                                  "ms_per_step": ms / a.steps, "sig_equal": sig == ref}), flush=True)


if __name__ == "__main__":
    main()
