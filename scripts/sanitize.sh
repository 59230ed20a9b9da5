#!/bin/bash
# compute-sanitizer over small runs of every kernel: memcheck, racecheck
# (shared memory of kernel T and its named barriers), synccheck.  usage: bash scripts/sanitize.sh <tag>
OUT=gpurun_out/${1:-san}
mkdir -p $OUT
cat > /tmp/san_run.py <<'PY'
import sys, numpy as np
sys.path.insert(0, ".")
import workloads, paper_conf_ipps_gavierrprs23_b200 as gs
kernel = sys.argv[1]
nl = workloads.synthetic(3000, 120, 16, 40, 12, seed=9, name="s")
prog = gs.Netlist.from_arrays(nl).compile()
lanes = 8192 if kernel == "df" else 16384 if kernel.startswith("lut_") else 2048
extra = {"lut_bulk": dict(flags=gs.GS_SIM_LUT_BULK, lane_groups=1),     # k_level_bulk (mbarrier ring)
         "lut_groups": dict(lane_groups=4),                              # concurrent graph branches
         "lut_hints": dict(flags=6, lane_groups=1, lut_unroll=4),        # L2-hinted stores + loads, U = 4
         "tile_global": dict(flags=gs.GS_SIM_TILE_SLOTS_GLOBAL, tile_words=4)}.get(kernel, {})
if kernel == "lut_hints":
    lanes = 65536
sim = gs.Sim(prog, lanes, kernel=kernel.split("_")[0], trace_words=[0, 5], trace_cycles=4,
             use_graphs=(kernel != "lut"), **extra)
sim.bind_generated(3)
sim.step(3)
if kernel in ("lut", "tile"):                # sub-batches: re-target, re-capture, step again
    sim.set_lane_offset(64 * 33)
    sim.step(2)
sim.read_outputs(); sim.read_registers(); sim.read_lane_signatures(); sim.signature()
sim.close()
print("ok", kernel)
PY
for k in ${KERNELS:-lut poly ab tile df lut_bulk lut_groups lut_hints tile_global}; do
  for tool in memcheck racecheck synccheck; do
    timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san_run.py $k > $OUT/${k}_${tool}.log 2>&1
    echo "$k $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $OUT/${k}_${tool}.log | tr '\n' ' ')" >> $OUT/summary.txt
  done
done
