#!/usr/bin/env python
"""Per-level issue efficiency of kernel A against level width, balance on / off (north_star:
"warp-issue efficiency on unbalanced layers"; PAPER.md P:44 — real circuits' unbalanced level
structure).

For one steady-state cycle of `bench.py --config <C> --lane-groups 1` (one launch per level, so
ncu's launches map 1:1 onto levels), ncu records every level launch: duration, SM issue-slot
utilisation (smsp__issue_active), warps active, grid and DRAM bytes.  The level widths come
from the compiled program (gs_program_level_widths, same compile options).  Writes one CSV per
(config, balance) under profiles/ and prints a summary line per run: time-weighted issue
efficiency, and the spread of level durations.

usage (GPU box):  python scripts/ncu_level_issue.py --tag r02 --config C4 C3
"""
import argparse
import csv
import io
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
METRICS = ("gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,"
           "sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,"
           "launch__grid_size")


def widths(cfg_name, balance):
    import workloads
    import paper_conf_ipps_gavierrprs23_b200 as gs
    nl = workloads.CONFIGS[cfg_name].netlist()
    prog = gs.Netlist.from_arrays(nl).compile(balance=balance)
    return [int(w) for w in prog.level_widths()]


def run(cfg_name, balance, tag):
    w = widths(cfg_name, balance)
    nonempty = [i for i, x in enumerate(w) if x]
    log = os.path.join(ROOT, "profiles", f"{tag}_level_issue_{cfg_name}_{'bal' if balance else 'asap'}.csv")
    cmd = ["ncu", "--metrics", METRICS, "--clock-control", "none", "-k", "regex:k_level_lut",
           "-s", str(len(nonempty)), "-c", str(len(nonempty)), "--csv", "--log-file", log,
           sys.executable, os.path.join(ROOT, "bench.py"), "--config", cfg_name, "--lane-groups", "1",
           "--quick", "--steps", "1", "--warmup", "1", "--cycles-per-step", "2"]
    if not balance:
        cmd.append("--no-balance")
    r = subprocess.run(cmd, capture_output=True, text=True, cwd=ROOT)
    if r.returncode != 0:
        sys.exit(r.stdout[-3000:] + r.stderr[-3000:])
    rows = list(csv.reader(io.StringIO("".join(ln for ln in open(log) if ln.startswith('"')))))
    hdr, rows = rows[0], rows[1:]
    ix = {h: i for i, h in enumerate(hdr)}
    per = {}
    for row in rows:
        per.setdefault(int(row[ix["ID"]]), {})[row[ix["Metric Name"]]] = float(row[ix["Metric Value"]].replace(",", ""))
    launches = [per[k] for k in sorted(per)]
    out = []
    for lvl, m in zip(nonempty, launches):
        out.append({"level": lvl + 1, "width": w[lvl], "us": m["gpu__time_duration.sum"] / 1e3,
                    "issue_active_pct": m["smsp__issue_active.avg.pct_of_peak_sustained_active"],
                    "warps_active_pct": m["sm__warps_active.avg.pct_of_peak_sustained_active"],
                    "grid": m["launch__grid_size"],
                    "dram_gbs": (m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]) / m["gpu__time_duration.sum"]})
    tab = os.path.join(ROOT, "profiles", f"{tag}_level_issue_{cfg_name}_{'bal' if balance else 'asap'}.jsonl")
    with open(tab, "w") as f:
        for o in out:
            f.write(json.dumps(o) + "\n")
    tot = sum(o["us"] for o in out)
    summ = {"config": cfg_name, "balance": balance, "levels": len(out),
            "width_min": min(o["width"] for o in out), "width_max": max(o["width"] for o in out),
            "width_cv": statistics.pstdev([o["width"] for o in out]) / statistics.mean([o["width"] for o in out]),
            "cycle_us_serialised": tot,
            "issue_active_time_weighted_pct": sum(o["issue_active_pct"] * o["us"] for o in out) / tot,
            "warps_active_time_weighted_pct": sum(o["warps_active_pct"] * o["us"] for o in out) / tot,
            "dram_gbs_time_weighted": sum(o["dram_gbs"] * o["us"] for o in out) / tot,
            "narrow_levels_share_of_time": sum(o["us"] for o in out if o["width"] < 1000) / tot,
            "table": os.path.relpath(tab, ROOT)}
    print(json.dumps(summ), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="r02")
    ap.add_argument("--config", nargs="+", default=["C4", "C3"])
    a = ap.parse_args()
    for c in a.config:
        for bal in (True, False):
            run(c, bal, a.tag)


if __name__ == "__main__":
    main()
