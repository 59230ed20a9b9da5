#!/usr/bin/env python
"""bench.py — stimulus·gate·cycle evaluations per second of the gsim hot path on B200.

Contract (see DESIGN.md §7 "Measurement"):
  python bench.py --gpus N --steps K --warmup W           (N > 1: under torch.distributed.run)
  python bench.py --impl reference ...                     (the CPU oracle arm, rank 0 only)

Default workload: BASELINE.json configs[4] (C5, the north_star's "largest config"): the
NVDLA-scale synthetic netlist (10M gates + 500k registers) over its whole batch of 262,144
stimuli for 100 cycles.  A *step* is that whole job: every lane of the batch simulated from
reset for 100 clock cycles through the whole hot path (stimulus generation, every level with
the fused register latch, the leftover latches and the output MISR).  The batch is STRONG-
scaled over the N ranks: rank r owns a contiguous 262,144/N-lane range (dist.shard) and runs
it as sequential sub-batches of at most --sub-lanes lanes in one workspace (the whole state
of C5 does not fit one GPU); every sub-batch starts from reset, so the all-reduced
lane_sig_sum is identical at every N (a self-check of the sharding).
`--config C4` (BASELINE configs[3], 1M gates, 65,536 lanes per GPU, weak-scaled) keeps the
round-1 shape: a step is --cycles-per-step cycles continuing from the previous step.

value = G_eval * lanes_total * cycles / max-over-ranks device time of the K timed steps.
"""
from __future__ import annotations

import argparse
import glob
import json
import os
import platform
import re
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "stimulus-gate-cycle evals/s at 1/2/4/8 B200; HBM GB/s vs roofline"
UNIT = "sgc/s"
DEFAULT_SUB_LANES = 32768       # sharded configs: lanes per sub-batch (tests use the same)
# level assignment per workload (bench --levels auto), from the round-2 A/B
# (profiles/r02_levels_ab.txt): the DRAM-bound configs run faster on ASAP levels (a producer
# and its readers stay closer in time, so more inputs hit L2: C4 +8 %, C5 +3 %), the
# launch-bound C3 on balanced levels (ASAP -8 %: narrow levels)
AUTO_LEVELS = {"C4": "asap", "C5": "asap"}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5")
    ap.add_argument("--cycles-per-step", type=int, default=0,
                    help="cycles per step (0 = the config's cycle count for sharded configs, else 100)")
    ap.add_argument("--sub-lanes", type=int, default=DEFAULT_SUB_LANES,
                    help="sharded configs: lanes per sub-batch (a multiple of the shard size / 2^k)")
    ap.add_argument("--lut-k", type=int, default=0, help="cone-collapse into <= L-input LUTs first")
    ap.add_argument("--lanes", type=int, default=0, help="override lanes per GPU (unsharded configs)")
    ap.add_argument("--kernel", default="lut", choices=["lut", "poly", "ab", "tile", "cluster", "auto"])
    ap.add_argument("--cluster-size", type=int, default=0, help="kernel C: CTAs per cluster (0 = auto)")
    ap.add_argument("--slab-lanes", type=int, default=0,
                    help="kernel C: lanes per slab (0 = auto); kernel A: lanes per slab of the segmented "
                         "slab schedule (0 = off)")
    ap.add_argument("--slab-min-gates", type=int, default=0,
                    help="kernel A slab schedule: narrowest level run per slab (0 = library default)")
    ap.add_argument("--levels", default="auto", choices=["auto", "balanced", "asap", "alap"],
                    help="level assignment (auto: the workload's measured best, DESIGN.md §6)")
    ap.add_argument("--no-balance", action="store_true", help="= --levels asap")
    ap.add_argument("--tile-words", type=int, default=0, help="kernel T: 32-bit words per slot")
    ap.add_argument("--tile-groups", type=int, default=0, help="kernel T: thread groups per CTA")
    ap.add_argument("--tile-desc", default="auto", choices=["auto", "tma", "global", "resident"],
                    help="kernel T descriptor source (auto: resident if it fits, else TMA stream)")
    ap.add_argument("--lut-unroll", type=int, default=0, help="vectors per thread (0 = auto)")
    ap.add_argument("--lane-groups", type=int, default=0,
                    help="kernel A: concurrent lane groups per cycle (0 = library auto, 1 = off)")
    ap.add_argument("--no-pdl", action="store_true", help="disable programmatic dependent launch")
    ap.add_argument("--no-grid-stride", action="store_true", help="kernel A: one CTA per work chunk")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend (gloo + --same-device: multi-rank test on one GPU)")
    ap.add_argument("--same-device", action="store_true",
                    help="test only: every rank uses cuda:0 (timings are NOT a scaling measurement)")
    ap.add_argument("--no-cpu-baseline", action="store_true", help="skip the oracle parity leg")
    ap.add_argument("--parity-lanes", type=int, default=256, help="oracle-checked lanes (parity leg)")
    ap.add_argument("--no-roofline", action="store_true")
    ap.add_argument("--core-seconds", type=float, default=12.0, help="target wall time of the 1-thread oracle leg")
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
        pw = [float(r[3]) for r in self.rows if len(r) > 3 and r[3].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, n in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "power_w_median": statistics.median(pw) if pw else None, "samples": len(self.rows)}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured (MEASURED_PEAKS.json)"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback (B200_PROFILING.md)"


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return platform.processor() or "unknown"


def insitu_traffic(key: str, build_id: str, program_hash: int):
    """In-situ DRAM bytes of one simulated cycle (ncu --graph-profiling graph of the cycle's
    CUDA graph, concurrency intact) from profiles/traffic.json — only if that entry was
    captured on THIS build of libgsim.so and THIS program; a stale entry is refused."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            e = json.load(f)["insitu"][key]
    except Exception:
        return None, f"no in-situ capture for {key}"
    if e.get("build_id") != build_id:
        return None, f"stale: captured on build {e.get('build_id')}, this is {build_id}"
    if int(e.get("program_hash", -1)) != int(program_hash):
        return None, "stale: captured on another program"
    return e, e.get("source")


# ------------------------------------------------------------------ CPU oracle legs
def oracle_parity_and_rate(nl, cfg, lanes_global, cycles, gpu_sigs, gpu_regs):
    """The parity leg (rank 0, N = 1): the oracle, as it stands, simulates the sampled lanes
    for exactly the GPU run's cycles (from reset, same seed); its per-lane MISR signatures and
    final registers are compared bit for bit with the GPU's.  Its wall time is the
    cpu_baseline rate (G x lanes x cycles / s) on all host threads."""
    import numpy as np
    import oracle
    threads = oracle.max_threads()
    G = int((nl.gate_k > 0).sum())
    t = time.perf_counter()
    o = oracle.simulate(nl, lanes_global, cycles, seed=cfg.stim_seed, threads=threads, want=("regs", "sig"))
    dt = time.perf_counter() - t
    sig_mm = int((o["sig"] != gpu_sigs).sum())
    reg_mm = int((o["regs"] != gpu_regs).sum()) if nl.n_reg else 0
    parity = {"lanes_checked": int(len(lanes_global)), "cycles": int(cycles),
              "registers_per_lane": int(nl.n_reg),
              "lane_signature_mismatches": sig_mm, "register_bit_mismatches": reg_mm,
              "mismatches": sig_mm + reg_mm,
              "what": "per-lane 64-bit MISR over every output of every cycle (R5) and every register "
                      "bit after the last cycle, oracle vs GPU, same netlist / seed / cycles from reset"}
    cpu = {"value": G * len(lanes_global) * cycles / dt, "unit": UNIT, "cores": threads, "kind": "oracle",
           "cpu_model": cpu_model(),
           "sample": f"{len(lanes_global)} lanes spread over every shard x {cycles} cycles of {cfg.name} "
                     f"(the parity leg), generated stimuli seed {cfg.stim_seed}; {dt:.1f} s wall on {threads} threads"}
    return parity, cpu


def oracle_per_core(nl, cfg, seconds: float):
    """--threads 1 figure: one lane on one thread for as many cycles as fit `seconds`."""
    import numpy as np
    import oracle
    G = int((nl.gate_k > 0).sum())
    t = time.perf_counter()
    oracle.simulate(nl, np.array([5]), 2, seed=cfg.stim_seed, threads=1, want=("sig",))
    per_cycle = max((time.perf_counter() - t) / 2, 1e-5)
    c = max(2, int(seconds / per_cycle))
    t = time.perf_counter()
    oracle.simulate(nl, np.array([5]), c, seed=cfg.stim_seed, threads=1, want=("sig",))
    dt = time.perf_counter() - t
    return {"value": G * c / dt, "unit": UNIT, "cores": 1, "sample": f"1 lane x {c} cycles, {dt:.1f} s"}


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
    # 16 lanes per thread: the oracle advances lanes in 16-lane blocks, one block per thread
    sample = np.linspace(0, cfg.lanes - 1, 16 * threads).astype(np.int64)
    cps = args.cycles_per_step or (cfg.cycles if cfg.shards > 1 else 100)
    # per step: every thread simulates one lane for c cycles from reset; size c so the whole
    # run is a few minutes
    t = time.perf_counter()
    oracle.simulate(nl, sample, 2, seed=cfg.stim_seed, threads=threads, want=("sig",))
    per_cycle = max((time.perf_counter() - t) / 2, 1e-4)
    budget = 150.0 / max(args.steps + args.warmup, 1)
    c = max(1, min(cps, int(budget / per_cycle)))
    for _ in range(args.warmup):
        oracle.simulate(nl, sample, c, seed=cfg.stim_seed, threads=threads, want=("sig",))
    t = time.perf_counter()
    for _ in range(args.steps):
        oracle.simulate(nl, sample, c, seed=cfg.stim_seed, threads=threads, want=("sig",))
    dt = time.perf_counter() - t
    val = G * len(sample) * c * args.steps / dt
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True,
            "scaling": "strong" if cfg.shards > 1 else "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic", "impl": "reference",
            "config": {"workload": f"{cfg.name}: {cfg.label}", "gates": G, "lanes_per_step": len(sample),
                       "cycles_per_step": c},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "cpu_model": cpu_model(),
                             "sample": f"{len(sample)} lanes x {c} cycles from reset per step of {cfg.name}"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def nccl_nranks(pattern: str):
    """nRanks that NCCL's INIT log reported for this process's communicator (None if absent)."""
    n = None
    for f in glob.glob(pattern):
        try:
            for ln in open(f, errors="replace"):
                m = re.search(r"nRanks\s+(\d+)", ln)
                if m:
                    n = int(m.group(1))
        except Exception:
            pass
    return n


# ------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    nccl_log = f"/tmp/gsim_nccl_{os.getpid()}.log"
    if world > 1 and args.dist_backend == "nccl":
        # NCCL INIT log to a file (never stdout: the driver reads one JSON line there)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", nccl_log)

    import numpy as np
    import torch
    import torch.distributed as dist
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    from paper_conf_ipps_gavierrprs23_b200 import dist as gdist

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
    sharded = cfg.shards > 1 and not args.lanes
    C = args.cycles_per_step or (cfg.cycles if sharded else 100)
    if sharded:
        # strong scaling: the whole batch is split over the ranks, each rank runs its range as
        # sub-batches (from reset every step) of at most --sub-lanes lanes
        lane_offset, lanes_rank = gdist.shard(cfg.lanes, world, rank)
        lanes = min(args.sub_lanes, lanes_rank)
        if lanes_rank % lanes:
            raise SystemExit(f"rank range {lanes_rank} is not a multiple of --sub-lanes {lanes}")
        subs = lanes_rank // lanes
    else:
        lanes = args.lanes or cfg.lanes
        lanes_rank, subs = lanes, 1
        lane_offset = rank * lanes                      # weak scaling: own global range per rank
    lanes_total = lanes_rank * world
    t0 = time.perf_counter()
    levels = "asap" if args.no_balance else args.levels
    if levels == "auto":
        levels = AUTO_LEVELS.get(cfg.name, "balanced")
    prog = gs.Netlist.from_arrays(nl).compile(balance={"balanced": 1, "asap": 0, "alap": 2}[levels],
                                              lut_k=args.lut_k)
    compile_s = time.perf_counter() - t0
    info = prog.info
    G = info["n_eval_gates"]
    if world > 1:
        gdist.check_same_program(info["program_hash"])
    stream = torch.cuda.Stream(device=local)
    flags = (8 if args.no_grid_stride else 0) | {"auto": 0, "global": 16, "tma": 32, "resident": 512}[args.tile_desc]
    sim = gs.Sim(prog, lanes, lane_offset=lane_offset, kernel=args.kernel, device=local, stream=stream,
                 lut_unroll=args.lut_unroll, pdl=not args.no_pdl, tile_words=args.tile_words,
                 tile_groups=args.tile_groups, lane_groups=args.lane_groups, flags=flags,
                 cluster_size=args.cluster_size, slab_lanes=args.slab_lanes,
                 slab_min_gates=args.slab_min_gates)
    sim.bind_generated(cfg.stim_seed)
    launches_per_cycle = sim.launches_per_cycle()

    def barrier():
        if world > 1:
            dist.barrier()

    sig_keys = ("lane_sig_sum", "out_popcount", "ab_mismatch", "invariant_violations")
    sub_sigs = []

    def one_step(record=None):
        """One step: sharded -> every sub-batch of this rank from reset for C cycles;
        otherwise C more cycles of the one sim.  record(j) is called after sub-batch j."""
        if not sharded:
            sim.step(C)
            return
        sub_sigs.clear()
        for j in range(subs):
            sim.set_lane_offset(lane_offset + j * lanes)      # re-targets and resets
            sim.step(C)
            sub_sigs.append(sim.signature())
            if record:
                record(j)

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
    if sharded:                        # the last timed step's sub-batches, summed mod 2^64
        sig = {k: (sum(d[k] for d in sub_sigs) % (1 << 64) if k in sig_keys else sig[k]) for k in sig}
    red = gdist.reduce_signature(sig) if world > 1 else sig
    cycles_per_rank_step = C * subs
    total_sgc = float(G) * lanes_total * C * args.steps
    value = total_sgc / (ms_max / 1e3)

    # ---------------------------------------------------------------- roofline (last sub-batch)
    roof = None
    pk, pk_src = peaks()
    if not args.no_roofline and not args.quick:
        ncyc = min(C, 10)
        pr = sim.profile_step(ncyc)
        achieved = pr["level_bytes"] / (pr["level_ms"] / 1e3) / 1e9
        per_launch_bytes = pr["level_bytes"] / max(pr["level_launches"], 1)
        groups = sim.config["lane_groups"]
        key = f"{cfg.name}:{lanes}:{args.kernel}:G{groups}"
        if args.kernel == "lut" and sim.launch.get("slab_lanes"):
            key += f":S{sim.launch['slab_lanes']}"
        tr, tr_src = insitu_traffic(key, gs.build_id(), info["program_hash"])
        ms_cycle = ms_max / (args.steps * cycles_per_rank_step)
        dram = None
        if tr:
            gbs = tr["dram_bytes_per_cycle"] / (ms_cycle / 1e3) / 1e9
            dram = {"bytes_per_cycle": tr["dram_bytes_per_cycle"], "read_bytes_per_cycle": tr.get("read_bytes"),
                    "write_bytes_per_cycle": tr.get("write_bytes"), "gbs": gbs, "frac": gbs / pk["hbm_gbs"],
                    "l2_hit_pct": tr.get("l2_hit_pct"), "source": tr_src,
                    "note": "actual DRAM bytes of one cycle (in-situ ncu graph capture of this build and "
                            "program) / this run's device time per cycle"}
        lvl_per_cycle = pr["level_launches"] / max(ncyc, 1)
        roof = {"bound": "hbm", "kernel": "k_level_lut_wide<4, false>" if args.kernel in ("lut", "auto") else args.kernel,
                "achieved": achieved, "peak": pk["hbm_gbs"], "unit": "GB/s", "frac": achieved / pk["hbm_gbs"],
                "frac_basis": "algorithmic gather-model bytes (k reads + 1 write + fused latch per gate-row) "
                              "/ measured HBM copy peak; L2 hits let it exceed the DRAM fraction, which is "
                              "dram_insitu.frac",
                "traffic": (tr["dram_bytes_per_cycle"] / lvl_per_cycle) if tr and lvl_per_cycle else None,
                "traffic_source": (f"in-situ DRAM bytes per cycle / {lvl_per_cycle:.0f} level launches per "
                                   f"cycle ({tr_src})") if tr else tr_src,
                "peak_source": f"hbm_gbs {pk_src}",
                "algorithmic_bytes_per_launch": per_launch_bytes,
                "level_share_of_step": pr["level_ms"] / pr["total_ms"],
                "lane_groups": groups, "lanes_per_launch": lanes // max(groups, 1),
                "dram_insitu": dram,
                "avg_level_launch_us": pr["level_ms"] * 1e3 / max(pr["level_launches"], 1),
                "measured": (f"CUDA events around every level launch on the sim stream, {ncyc} un-graphed "
                             f"cycles of the last sub-batch after the timed region") if groups == 1 else
                            (f"{groups} lane groups run their level chains concurrently: timing-event graph "
                             f"nodes at the fork and join of the level region of each of {ncyc} graph-replayed "
                             f"cycles after the timed region; achieved = algorithmic bytes of all level "
                             f"launches / region time, avg_level_launch_us = region time / launches")}

    # ---------------------------------------------------------------- e2e
    # paper-style: every step streams its stimuli host->device and EVERY output of
    # every cycle device->host (gs_sim_run_streamed: pinned buffers, chunks overlapped with
    # compute on a copy stream), all inside the timed region
    e2e = None
    if not args.no_e2e and not args.quick:
        n_pi, n_po = info["n_pi"], info["n_po"]
        words = lanes // 64
        K2 = max(1, min(args.steps, 2))
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
                if sharded:
                    sim.set_lane_offset(lane_offset + j * lanes)
                sim.run_streamed(h_np, o_np)
        e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1)
        ems = gdist.max_over_ranks(ems) if world > 1 else ems
        e2e = {"value": float(G) * lanes_total * C * K2 / (ems / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(host.numel() * 8) * subs, "d2h_bytes_per_step": int(out_buf.numel() * 8) * subs,
               "steps": K2, "path": "gs_sim_run_streamed: pinned host stimuli in, every output of every "
                                    "cycle out, 25-cycle chunks overlapped with compute"
                                    + ("; every sub-batch from reset" if sharded else "")}
        sim.bind_generated(cfg.stim_seed)

    # ---------------------------------------------------------------- parity leg + cpu baseline
    cpu, parity = None, None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.quick:
        # a verification pass identical to a timed step's work (every sub-batch from reset
        # for the config's cycles), reading back per-lane signatures and registers, then the
        # oracle on the sampled lanes
        vc = cfg.cycles
        sample = workloads.sample_lanes(lanes_total, max(cfg.shards, 1) if sharded else 1,
                                        args.parity_lanes // (cfg.shards if sharded else 1), seed=2,
                                        groups=max(sim.config["lane_groups"], 1),
                                        lanes_per_word=2 if sharded else 4)
        sample = sample[(sample >= lane_offset) & (sample < lane_offset + lanes_rank)]
        gsig = np.zeros(len(sample), dtype=np.uint64)
        greg = np.zeros((len(sample), info["n_reg"]), dtype=np.uint8)

        def record(j):
            lo = lane_offset + j * lanes
            m = (sample >= lo) & (sample < lo + lanes)
            if not m.any():
                return
            loc = sample[m] - lo
            gsig[m] = sim.read_lane_signatures()[loc]
            if info["n_reg"]:                 # [reg][word] -> the sampled lanes' bits only
                w = sim.read_registers()[:, loc // 64]
                greg[m] = ((w >> (loc % 64).astype(np.uint64)[None, :]) & np.uint64(1)).astype(np.uint8).T
        t = time.perf_counter()
        for j in range(subs):
            sim.set_lane_offset(lane_offset + j * lanes)
            sim.step(vc)
            record(j)
        vdt = time.perf_counter() - t
        parity, cpu = oracle_parity_and_rate(nl, cfg, sample, vc, gsig, greg)
        parity["gpu_verification_pass_s"] = round(vdt, 2)
        cpu["per_core"] = oracle_per_core(nl, cfg, args.core_seconds)

    if rank == 0:
        nranks = nccl_nranks(nccl_log) if world > 1 and args.dist_backend == "nccl" else None
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
            "scaling": "strong" if sharded else "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic",
            "config": {"workload": f"{cfg.name}: {cfg.label}", "gates": G, "registers": info["n_reg"],
                       "levels": info["n_levels"], "lanes_total": lanes_total, "lanes_per_gpu": lanes_rank,
                       "sub_batches_per_gpu": subs, "lanes_per_sub_batch": lanes,
                       "cycles_per_step": C, "kernel": args.kernel, "level_assignment": levels,
                       "lut_unroll": args.lut_unroll, "lane_groups": sim.config["lane_groups"],
                       "pdl": not args.no_pdl, "tile_words": args.tile_words, "tile_groups": args.tile_groups,
                       "lut_k": args.lut_k, "grid_stride": not args.no_grid_stride,
                       "launch": sim.launch,
                       "l2": "inputs larger than L2 (state %.1f GB per sub-batch)" % (info["n_rows"] * lanes / 8 / 1e9),
                       "step": (f"the whole batch: {subs} sub-batch(es) of {lanes} lanes per GPU, each from reset "
                                f"for {C} cycles" if sharded else f"{C} more cycles over every lane of the GPU"),
                       "parallelism": f"dp{world} (stimulus sharding)" + (" TEST: all ranks on cuda:0"
                                                                              if args.same_device else ""),
                       "compile_s": round(compile_s, 2), "build_id": gs.build_id(),
                       "program_hash": str(info["program_hash"]),
                       "paper_style_gcps": value * (G + info["n_reg"]) / G},
            # per cycle: stim + level launches + end-of-cycle (kernels T / C: one launch per step);
            # sharded: per sub-batch also the reset's 3 row fills and the signature's k_lane_sigs
            "gpu_launches": int(args.steps * subs * (launches_per_cycle * (1 if args.kernel in ("tile", "cluster") else C)
                                                     + (4 if sharded else 0))),
            "signature": {k: str(v) for k, v in red.items()},
            "nccl": ({"nranks": nranks, "ok": nranks == world} if nranks is not None else None),
            "clocks": clk,
            "roofline": roof,
            "parity": parity,
            "cpu_baseline": cpu,
            "e2e": e2e,
        }
        print(json.dumps(line), flush=True)
    sim.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
