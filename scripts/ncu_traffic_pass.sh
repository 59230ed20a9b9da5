#!/bin/bash
# ncu metrics-only pass over every level launch of one steady-state cycle of the bench
# command for config $1 (extra bench args after it); writes gpurun_out/traffic_$1.csv.
# Then, here: python scripts/ncu_cycle_traffic.py gpurun_out/traffic_<cfg>.csv "<key>" <source>
CFG=$1; shift
L=$(python - "$CFG" "$@" <<'PY'
import sys, workloads, paper_conf_ipps_gavierrprs23_b200 as gs
cfg = workloads.CONFIGS[sys.argv[1]]
prog = gs.Netlist.from_arrays(cfg.netlist()).compile()
lanes = cfg.lanes // getattr(cfg, "shards", 1)
args = sys.argv[2:]
g = int(args[args.index("--lane-groups") + 1]) if "--lane-groups" in args else 0
sim = gs.Sim(prog, lanes, kernel="lut", lane_groups=g)
print(sim.launches_per_cycle() - 2)
PY
)
mkdir -p gpurun_out
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:k_level_lut -s $L -c $L --csv --log-file gpurun_out/traffic_$CFG.csv \
    python bench.py --config $CFG --quick --steps 1 --warmup 1 --cycles-per-step 1 "$@" > gpurun_out/traffic_$CFG.log 2>&1
echo "levels per cycle $L rc=$?" >> gpurun_out/traffic_$CFG.log
