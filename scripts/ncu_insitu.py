#!/usr/bin/env python
"""In-situ DRAM traffic of one simulated cycle, keyed to the build (bench.py roofline.dram_insitu).

Runs `bench.py <args> --quick` under `ncu --graph-profiling graph` (each cycle's CUDA graph is
measured as ONE workload, so the concurrent lane-group branches and the L2 reuse between
level launches are intact; caches are flushed only before each graph), takes the median
DRAM read / write bytes over the captured cycle graphs, and stores them in
profiles/traffic.json under "insitu"[<config>:<lanes per sub-batch>:<kernel>:G<lane groups>]
together with the gs_build_id() and program hash of the run.  bench.py uses an entry only
if both match the benched build and program.

usage (on a GPU box):  python scripts/ncu_insitu.py --tag r02 -- --config C5
"""
import argparse
import csv
import io
import json
import os
import shutil
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="r02")
    ap.add_argument("--count", type=int, default=48, help="ncu -c (kernels + graphs profiled)")
    ap.add_argument("bench_args", nargs=argparse.REMAINDER)
    a = ap.parse_args()
    bargs = [x for x in a.bench_args if x != "--"]
    out_dir = os.path.join(ROOT, "gpurun_out", "insitu")
    os.makedirs(out_dir, exist_ok=True)
    name = "_".join(x.strip("-") for x in bargs) or "default"
    log = os.path.join(out_dir, f"{a.tag}_{name}.csv")
    cmd = ["ncu", "--graph-profiling", "graph", "--metrics", METRICS, "--clock-control", "none",
           "-c", str(a.count), "--csv", "--log-file", log, sys.executable, os.path.join(ROOT, "bench.py"),
           *bargs, "--quick", "--steps", "1", "--warmup", "1", "--cycles-per-step", "3"]
    r = subprocess.run(cmd, capture_output=True, text=True, cwd=ROOT)
    line = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    if r.returncode != 0 or not line:
        sys.exit(f"bench under ncu failed rc={r.returncode}\n{r.stdout[-2000:]}\n{r.stderr[-2000:]}")
    b = json.loads(line[-1])
    cfg = b["config"]
    rows = list(csv.reader(io.StringIO("".join(ln for ln in open(log) if ln.startswith('"')))))
    hdr, rows = rows[0], rows[1:]
    ix = {h: i for i, h in enumerate(hdr)}
    graphs = {}
    for row in rows:
        if row[ix["Kernel Name"]] != "graph":
            continue
        graphs.setdefault(row[ix["ID"]], {})[row[ix["Metric Name"]]] = float(row[ix["Metric Value"]].replace(",", ""))
    vals = [g for g in graphs.values() if "dram__bytes_read.sum" in g]
    if len(vals) < 2:
        sys.exit(f"only {len(vals)} cycle graphs captured")
    vals = vals[1:]                                      # skip the very first (cold program upload)
    rd = statistics.median(v["dram__bytes_read.sum"] for v in vals)
    wr = statistics.median(v["dram__bytes_write.sum"] for v in vals)
    t_ns = statistics.median(v["gpu__time_duration.sum"] for v in vals)
    hit = statistics.median(v["lts__t_sector_hit_rate.pct"] for v in vals)
    key = f"{cfg['workload'].split(':')[0]}:{cfg['lanes_per_sub_batch']}:{cfg['kernel']}:G{cfg['lane_groups']}"
    if cfg["kernel"] == "lut" and cfg.get("launch", {}).get("slab_lanes"):
        key += f":S{cfg['launch']['slab_lanes']}"     # kernel A segmented slab schedule
    entry = {"dram_bytes_per_cycle": rd + wr, "read_bytes": rd, "write_bytes": wr, "l2_hit_pct": hit,
             "ncu_graph_us": t_ns / 1e3, "graphs": len(vals), "build_id": cfg["build_id"],
             "program_hash": cfg["program_hash"], "bench_args": " ".join(bargs),
             "source": f"ncu --graph-profiling graph, median of {len(vals)} cycle graphs "
                       f"(profiles/{a.tag}_insitu_{name}.csv)"}
    shutil.copy(log, os.path.join(ROOT, "profiles", f"{a.tag}_insitu_{name}.csv"))
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        d = json.load(open(tpath))
    except Exception:
        d = {}
    d.setdefault("insitu", {})[key] = entry
    d["note"] = ("insitu: DRAM bytes of one simulated cycle measured in situ (ncu --graph-profiling graph) "
                 "by scripts/ncu_insitu.py, keyed <config>:<lanes>:<kernel>:G<groups> and tagged with the "
                 "gs_build_id() / program hash they were captured on; bench.py refuses stale entries")
    json.dump(d, open(tpath, "w"), indent=1)
    print(json.dumps({key: entry}))


if __name__ == "__main__":
    main()
