#!/usr/bin/env python
"""Summarise a gpurun ncu launch list (--metrics gpu__time_duration.sum) and an ncu --set full
report into plain-text files for profiles/.

usage: python scripts/ncu_summary.py <launches.csv> <prof.ncu-rep> <out_prefix>
"""
import collections
import csv
import io
import subprocess
import sys

KEYS = ["Kernel Name", "Grid Size", "Block Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__occupancy_limit_registers",
        "sm__maximum_warps_per_active_cycle_pct", "lts__t_bytes.sum", "l1tex__t_bytes.sum",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio"]


def launches(path):
    rows = list(csv.reader(open(path)))
    i = [j for j, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr, data = rows[i], rows[i + 1:]
    kn, mv, mu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in data:
        if len(r) <= mv:
            continue
        v = float(r[mv].replace(",", "")) * scale.get(r[mu], 1.0)
        name = r[kn].split("(")[0]
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(a[1] for a in agg.values())
    out = [f"# ncu launch list ({path}); per-launch device time, cold-cache, serialised",
           f"# {'kernel':45s} launches   total_us    share    avg_us"]
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"{k:47s} {n:6d} {t:10.1f} {t / tot:8.3f} {t / n:9.2f}")
    return "\n".join(out) + "\n"


def traffic(path):
    """Mean dram read+write bytes per profiled launch, per kernel (for bench.py roofline.traffic)."""
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    acc = collections.defaultdict(list)
    for r in rows[2:]:
        b = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = hdr.index(k)
            b += float(r[i].replace(",", "")) * mult[units[i]]
        t = float(r[hdr.index("gpu__time_duration.sum")].replace(",", ""))
        acc[r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "")].append((b, t))
    return {k: {"traffic_bytes_per_launch": sum(b for b, _ in v) / len(v),
                "ncu_us_per_launch": sum(t for _, t in v) / len(v), "launches": len(v)}
            for k, v in acc.items()}


def full(path):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    out = [f"# ncu --set full ({path}); one block per profiled launch"]
    for r in rows[2:]:
        out.append("---")
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                out.append(f"{k:75s} {units[i]:>14s} {r[i]}")
    return "\n".join(out) + "\n"


if __name__ == "__main__":
    lc, rep, pre = sys.argv[1:4]
    if lc != "-":
        open(pre + "_launches.txt", "w").write(launches(lc))
    if rep != "-":
        open(pre + "_full.txt", "w").write(full(rep))
        import json
        json.dump({"source": pre + "_full.txt", "kernels": traffic(rep)},
                  open(pre + "_traffic.json", "w"), indent=1)
