#!/usr/bin/env python
"""Average DRAM traffic per level launch over ONE whole simulated cycle, from an ncu
metrics-only pass, merged into profiles/traffic.json (bench.py's roofline.traffic).

The capture (one GPU, under gpurun), skipping the first cycle's level launches:
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --clock-control none -k regex:k_level_lut -s <L> -c <L> --csv --log-file <csv> \
      python bench.py --config C4 --quick --steps 1 --warmup 1 --cycles-per-step 1
with L = level launches per cycle (non-empty levels x lane groups).

usage: python scripts/ncu_cycle_traffic.py <csv> <key> <source-name>
  key e.g. "C4:k_level_lut_wide<4, 0>:G4"
"""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def parse(path):
    rows = list(csv.reader(open(path)))
    i = [j for j, r in enumerate(rows) if "Kernel Name" in r and "Metric Name" in r][0]
    hdr = rows[i]
    kn, idx, mn, mv, mu = (hdr.index("Kernel Name"), hdr.index("ID"), hdr.index("Metric Name"),
                           hdr.index("Metric Value"), hdr.index("Metric Unit"))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1.0,
             "msecond": 1e3, "ns": 1e-3, "us": 1.0, "ms": 1e3}
    launches = collections.defaultdict(dict)
    for r in rows[i + 1:]:
        if len(r) <= mv:
            continue
        launches[r[idx]][r[mn]] = float(r[mv].replace(",", "")) * scale.get(r[mu], 1.0)
        launches[r[idx]]["name"] = r[kn].split("(")[0]
    return list(launches.values())


def main():
    path, key, src = sys.argv[1], sys.argv[2], sys.argv[3]
    ls = parse(path)
    n = len(ls)
    rd = sum(x["dram__bytes_read.sum"] for x in ls)
    wr = sum(x["dram__bytes_write.sum"] for x in ls)
    us = sum(x["gpu__time_duration.sum"] for x in ls)
    names = collections.Counter(x["name"] for x in ls)
    tj = os.path.join(ROOT, "profiles", "traffic.json")
    d = json.load(open(tj))
    d["kernels"][key] = {"traffic_bytes_per_launch": (rd + wr) / n, "dram_read_bytes_cycle": rd,
                         "dram_write_bytes_cycle": wr, "ncu_us_per_launch": us / n, "launches": n,
                         "kernels": dict(names), "source": src,
                         "how": "ncu metrics-only pass over every level launch of one cycle "
                                "(cold-cache, serialised), averaged per launch"}
    json.dump(d, open(tj, "w"), indent=1)
    print(key, json.dumps(d["kernels"][key]))


if __name__ == "__main__":
    main()
