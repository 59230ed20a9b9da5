#!/usr/bin/env python
"""bench.py — stimulus·gate·cycle evaluations per second of the gsim hot path on B200.

Contract:
  python bench.py --gpus N --steps K --warmup W           (N > 1: under torch.distributed.run)
  python bench.py --impl reference ...                     (the CPU oracle arm, rank 0 only)

A *step* is ``--cycles-per-step`` clock cycles (default 100) of the whole hot path —
stimulus generation, every level of gates with the fused register latch, the remaining
latches and the output MISR — over one batch of stimuli.  The default workload is
BASELINE.json configs[3] (C4: RISC-V-core-scale synthetic, 1M gates + 50k registers,
65,536 stimuli per GPU), the largest configuration that fits one GPU; its 1,000-cycle
run is 10 steps.  Multi-GPU is weak scaling: every rank simulates its own 65,536 global
lanes (lane_offset = rank * lanes) of the same netlist; the only collective is the
all-reduce of the per-rank signatures.  C5 (BASELINE configs[4], 8 shards of 32,768 lanes)
runs its whole 262,144-lane batch at any N dividing 8: each rank simulates 8/N shards as
sequential sub-batches in one workspace (gs_sim_set_lane_offset); a step is then C cycles of
every sub-batch, each from reset.

value = G_eval * lanes_total * cycles / max-over-ranks device time of the K timed steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "stimulus-gate-cycle evals/s at 1/2/4/8 B200; HBM GB/s vs roofline"
UNIT = "sgc/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4")
    ap.add_argument("--cycles-per-step", type=int, default=100)
    ap.add_argument("--lut-k", type=int, default=0, help="cone-collapse into <= L-input LUTs first")
    ap.add_argument("--order", type=int, default=0, help="gate order inside a level (0 by k/id, 1 recency)")
    ap.add_argument("--lanes", type=int, default=0, help="override lanes per GPU")
    ap.add_argument("--kernel", default="lut", choices=["lut", "poly", "ab", "df", "tile"])
    ap.add_argument("--tile-words", type=int, default=0, help="kernel T: 32-bit words per slot")
    ap.add_argument("--tile-groups", type=int, default=0, help="kernel T: thread groups per CTA")
    ap.add_argument("--tile-slots-global", action="store_true",
                    help="kernel T: live slots in the workspace (L1/L2) instead of shared memory")
    ap.add_argument("--df-interleave", type=int, default=0, help="kernel D: slabs walked together")
    ap.add_argument("--df-gpw", type=int, default=0, help="kernel D: gates per warp per item")
    ap.add_argument("--lane-slabs", type=int, default=0, help="L2 lane slabs (0 = library default)")
    ap.add_argument("--lut-unroll", type=int, default=0, help="vectors per thread (0 = auto)")
    ap.add_argument("--lane-groups", type=int, default=0,
                    help="kernel A: concurrent lane groups per cycle (0 = library auto, 1 = off)")
    ap.add_argument("--no-pdl", action="store_true", help="disable programmatic dependent launch")
    ap.add_argument("--no-grid-stride", action="store_true", help="kernel A: one CTA per work chunk")
    ap.add_argument("--l2-hints", type=int, default=0, help="kernel A L2 hints: 0 off, 1 stores, 2 +loads")
    ap.add_argument("--lut-bulk", default="auto", choices=["auto", "on", "off"],
                    help="kernel A bulk-copy staged gathers (auto = library default: off)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend (gloo + --same-device: multi-rank test on one GPU)")
    ap.add_argument("--same-device", action="store_true",
                    help="test only: every rank uses cuda:0 (timings are NOT a scaling measurement)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-roofline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=25.0, help="target oracle wall time (calibrated)")
    ap.add_argument("--quick", action="store_true", help="ncu mode: no e2e/cpu/roofline/clocks")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled DURING the timed region (200 ms)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm = [float(r[1]) for r in self.rows if len(r) > 2 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, n in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(self.rows)}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback"


KERNEL_NAMES = {"lut": "k_level_lut_wide<4, 0>", "df": "k_dataflow<1>", "poly": "k_level_poly",
                "ab": "k_level_lut_wide<4, 0>", "tile": "k_tile"}


def ncu_traffic(config: str, kernel: str):
    """dram read+write bytes per launch of `kernel` on `config` from the committed ncu --set
    full summary (profiles/traffic.json, from scripts/ncu_summary.py on the same bench command)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            d = json.load(f)
        e = d["kernels"][f"{config}:{kernel}"]
        return {"traffic_bytes_per_launch": e["traffic_bytes_per_launch"],
                "source": e.get("source", d.get("source"))}
    except Exception:
        return None


def insitu_dram(config: str, groups: int, ms_per_cycle: float, peak: float):
    """Actual DRAM rate of the whole cycle: the committed in-situ DRAM bytes of one cycle graph
    (ncu --graph-profiling graph, profiles/traffic.json 'cycles') / this run's time per cycle."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            e = json.load(f)["cycles"][f"{config}:G{groups}"]
    except Exception:
        return None
    gbs = e["dram_bytes_per_cycle"] / (ms_per_cycle / 1e3) / 1e9
    return {"bytes_per_cycle": e["dram_bytes_per_cycle"], "gbs": gbs, "frac": gbs / peak, "source": e["source"]}


# ------------------------------------------------------------------ CPU oracle
def oracle_rate(nl, cfg, lane_offset, seconds: float, cycles_cap: int | None = None):
    """Time the oracle (as it stands) on a bounded sample: n_threads lanes x c cycles."""
    import numpy as np
    import oracle
    threads = oracle.max_threads()
    G = int((nl.gate_k > 0).sum())
    lanes_total = cfg.lanes
    # calibration: one lane per thread, 8 cycles
    sample = np.linspace(0, lanes_total - 1, threads).astype(np.int64) + lane_offset
    t = time.perf_counter()
    oracle.simulate(nl, sample, 8, seed=cfg.stim_seed, threads=threads, want=("sig",))
    dt = max(time.perf_counter() - t, 1e-3)
    per_cycle = dt / 8
    cycles = max(2, int(seconds / per_cycle))
    if cycles_cap:
        cycles = min(cycles, cycles_cap)
    t = time.perf_counter()
    oracle.simulate(nl, sample, cycles, seed=cfg.stim_seed, threads=threads, want=("sig",))
    dt = time.perf_counter() - t
    return {"value": G * len(sample) * cycles / dt, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"{len(sample)} lanes (one per thread, spread over the batch) x {cycles} cycles "
                      f"of {cfg.name}, generated stimuli seed {cfg.stim_seed}; {dt:.1f} s wall"}, dt


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, rank 0 only, same metric/config."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np
    import oracle
    import workloads
    cfg = workloads.CONFIGS[args.config]
    nl = cfg.netlist()
    G = int((nl.gate_k > 0).sum())
    threads = oracle.max_threads()
    sample = np.linspace(0, cfg.lanes - 1, threads).astype(np.int64)
    # per step: every thread simulates one lane for c cycles; size c so the run is minutes
    t = time.perf_counter()
    oracle.simulate(nl, sample, 2, seed=cfg.stim_seed, threads=threads, want=("sig",))
    per_cycle = max((time.perf_counter() - t) / 2, 1e-4)
    budget = 150.0 / max(args.steps + args.warmup, 1)
    c = max(1, min(args.cycles_per_step, int(budget / per_cycle)))
    for _ in range(args.warmup):
        oracle.simulate(nl, sample, c, seed=cfg.stim_seed, threads=threads, want=("sig",))
    t = time.perf_counter()
    for _ in range(args.steps):
        oracle.simulate(nl, sample, c, seed=cfg.stim_seed, threads=threads, want=("sig",))
    dt = time.perf_counter() - t
    val = G * len(sample) * c * args.steps / dt
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": f"{cfg.name}: {cfg.label}", "gates": G, "lanes_per_step": len(sample),
                       "cycles_per_step": c},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"{len(sample)} lanes x {c} cycles per step of {cfg.name}"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import torch.distributed as dist
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    from paper_conf_ipps_gavierrprs23_b200 import dist as gdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        print(f"warning: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
    if args.same_device:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")

    cfg = workloads.CONFIGS[args.config]
    nl = cfg.netlist()
    # lanes = one sim's lanes; a sharded config (C5: 8 shards of 32,768 lanes) gives every rank
    # shards/world of them, run as sequential sub-batches in one workspace
    lanes = args.lanes or (cfg.lanes // cfg.shards if cfg.shards > 1 else cfg.lanes)
    subs = cfg.shards // world if (not args.lanes and cfg.shards > world and cfg.shards % world == 0) else 1
    lanes_rank = lanes * subs
    lane_offset = rank * lanes_rank
    t0 = time.perf_counter()
    prog = gs.Netlist.from_arrays(nl).compile(balance=True, lut_k=args.lut_k, order=args.order)
    compile_s = time.perf_counter() - t0
    info = prog.info
    G = info["n_eval_gates"]
    if world > 1:
        gdist.check_same_program(info["program_hash"])
    stream = torch.cuda.Stream(device=local)
    sim = gs.Sim(prog, lanes, lane_offset=lane_offset, kernel=args.kernel, device=local, stream=stream,
                 lane_slabs=args.lane_slabs, lut_unroll=args.lut_unroll,
                 df_interleave=args.df_interleave, df_gates_per_warp=args.df_gpw, pdl=not args.no_pdl,
                 tile_words=args.tile_words, tile_groups=args.tile_groups, lane_groups=args.lane_groups,
                 flags=(2 if args.l2_hints >= 1 else 0) | (4 if args.l2_hints >= 2 else 0) |
                 (8 if args.no_grid_stride else 0) | (256 if args.tile_slots_global else 0) |
                 {"auto": 0, "on": 64, "off": 128}[args.lut_bulk])
    sim.bind_generated(cfg.stim_seed)
    C = args.cycles_per_step
    launches_per_cycle = sim.launches_per_cycle()

    def barrier():
        if world > 1:
            dist.barrier()

    sig_keys = ("lane_sig_sum", "out_popcount", "ab_mismatch", "invariant_violations")
    sub_sigs = []

    def one_step():
        """C cycles over this rank's whole batch: one sim, or every sub-batch from reset."""
        if subs == 1:
            sim.step(C)
            return
        sub_sigs.clear()
        for j in range(subs):
            sim.set_lane_offset(lane_offset + j * lanes)      # syncs, re-targets, resets
            sim.step(C)
            sub_sigs.append(sim.signature())

    for _ in range(args.warmup):
        one_step()
    sim.sync()
    torch.cuda.synchronize()
    barrier()
    clocks = ClockSampler(local)
    if not args.quick:
        clocks.start()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        one_step()
    ev1.record(stream)
    torch.cuda.synchronize()
    clk = clocks.stop() if not args.quick else None
    ms = ev0.elapsed_time(ev1)
    barrier()
    ms_max = gdist.max_over_ranks(ms) if world > 1 else ms
    sig = sim.signature()
    if subs > 1:                       # the last timed step's sub-batches, summed mod 2^64
        sig = {k: (sum(d[k] for d in sub_sigs) % (1 << 64) if k in sig_keys else sig[k]) for k in sig}
    red = gdist.reduce_signature(sig) if world > 1 else sig

    total_sgc = float(G) * lanes_rank * world * C * args.steps
    value = total_sgc / (ms_max / 1e3)

    # ---------------------------------------------------------------- roofline
    roof = None
    pk, pk_src = peaks()
    if not args.no_roofline and not args.quick:
        pr = sim.profile_step(min(C, 10))
        achieved = pr["level_bytes"] / (pr["level_ms"] / 1e3) / 1e9
        per_launch_bytes = pr["level_bytes"] / max(pr["level_launches"], 1)
        kname = KERNEL_NAMES[args.kernel]
        if args.kernel == "df":
            kname = f"k_dataflow<{lanes // (args.lane_slabs or lanes // 4096) // 4096}>"
        G_groups = sim.config["lane_groups"]
        tr = ncu_traffic(args.config, f"{kname}:G{G_groups}")
        roof = {"bound": "hbm", "kernel": kname,
                "achieved": achieved, "peak": pk["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / pk["hbm_gbs"],
                "traffic": tr["traffic_bytes_per_launch"] if tr else None,
                "traffic_source": tr["source"] if tr else None,
                "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({pk_src})",
                "algorithmic_bytes_per_launch": per_launch_bytes,
                "level_share_of_step": pr["level_ms"] / pr["total_ms"],
                "lane_groups": G_groups,
                "dram_insitu": insitu_dram(args.config, G_groups, ms_max / (args.steps * C * subs), pk["hbm_gbs"]),
                "avg_level_launch_us": pr["level_ms"] * 1e3 / max(pr["level_launches"], 1),
                "measured": (f"CUDA events around every level launch on the sim stream, "
                             f"{min(C, 10)} un-graphed cycles after the timed region") if G_groups == 1 else
                            (f"{G_groups} lane groups run their level chains concurrently: timing-event "
                             f"graph nodes at the fork and join of the level region of each of {min(C, 10)} "
                             f"graph-replayed cycles after the timed region; achieved = algorithmic bytes "
                             f"of all level launches / region time, avg_level_launch_us = region time / "
                             f"launches (launches overlap)")}

    # ---------------------------------------------------------------- e2e
    # paper-style: every step streams its stimuli host->device and EVERY output of
    # every cycle device->host (gs_sim_run_streamed: pinned buffers, chunks overlapped with
    # compute on a copy stream), all inside the timed region
    e2e = None
    if not args.no_e2e and not args.quick:
        n_pi, n_po = info["n_pi"], info["n_po"]
        words = lanes // 64
        K2 = max(1, min(args.steps, 3))
        host = torch.empty((C, n_pi, words), dtype=torch.int64).pin_memory()
        host.random_()
        h_np = host.numpy().view(np.uint64)
        out_buf = torch.empty((C, n_po, words), dtype=torch.int64).pin_memory()
        o_np = out_buf.numpy().view(np.uint64)
        sim.reset()
        sim.run_streamed(h_np, o_np)             # warm-up: allocates the staging buffers
        sim.sync()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(K2):
            for j in range(subs):
                if subs > 1:
                    sim.set_lane_offset(lane_offset + j * lanes)
                sim.run_streamed(h_np, o_np)
        e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1)
        ems = gdist.max_over_ranks(ems) if world > 1 else ems
        e2e = {"value": float(G) * lanes_rank * world * C * K2 / (ems / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(host.numel() * 8) * subs, "d2h_bytes_per_step": int(out_buf.numel() * 8) * subs,
               "steps": K2, "path": "gs_sim_run_streamed: pinned host stimuli in, every output of every "
                                    "cycle out, 25-cycle chunks overlapped with compute"}

    # ---------------------------------------------------------------- cpu baseline
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.quick:
        cpu, _ = oracle_rate(nl, cfg, lane_offset, args.cpu_seconds, cycles_cap=None)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
            "config": {"workload": f"{cfg.name}: {cfg.label}", "gates": G, "registers": info["n_reg"],
                       "levels": info["n_levels"], "lanes_per_gpu": lanes_rank, "lanes_total": lanes_rank * world,
                       "sub_batches_per_gpu": subs, "lanes_per_sub_batch": lanes,
                       "cycles_per_step": C, "kernel": args.kernel, "balance": True,
                       "lane_slabs": args.lane_slabs, "lut_unroll": args.lut_unroll,
                       "lane_groups": sim.config["lane_groups"],
                       "df_interleave": args.df_interleave, "df_gpw": args.df_gpw,
                       "pdl": not args.no_pdl, "tile_words": args.tile_words,
                       "tile_groups": args.tile_groups, "tile_slots_global": args.tile_slots_global,
                       "l2_hints": args.l2_hints, "lut_k": args.lut_k, "order": args.order,
                       "grid_stride": not args.no_grid_stride,
                       "l2": "inputs larger than L2 (state %.1f GB per GPU)" % (info["n_rows"] * lanes / 8 / 1e9),
                       "step": f"{C} cycles over every lane of the GPU" + (
                           f" ({subs} sub-batches of {lanes} lanes, each from reset)" if subs > 1 else ""),
                       "parallelism": f"dp{world} (stimulus sharding)" + (" TEST: all ranks on cuda:0"
                                                                              if args.same_device else ""),
                       "compile_s": round(compile_s, 2),
                       "paper_style_gcps": value * (G + info["n_reg"]) / G},
            "gpu_launches": int(launches_per_cycle * (1 if args.kernel == "tile" else C) * args.steps * subs),
            "signature": {k: str(v) for k, v in red.items()},
            "clocks": clk,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
        }
        print(json.dumps(line), flush=True)
    sim.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
