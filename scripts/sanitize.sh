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
if kernel.startswith("tile_narrow"):                 # k <= 2, no registers: 8-byte descriptors
    nl = workloads.array_multiplier(12)
prog = gs.Netlist.from_arrays(nl).compile()
lanes = 16384 if kernel.startswith("lut_") else 2048
extra = {"lut_groups": dict(lane_groups=4),                              # concurrent graph branches
         "lut_u4": dict(lane_groups=1, lut_unroll=4),                    # U = 4 wide path
         "tile_tma": dict(flags=gs.GS_SIM_TILE_DESC_TMA, tile_groups=2),  # chunked TMA stream, 2 groups
         "tile_global": dict(flags=gs.GS_SIM_TILE_DESC_GLOBAL, tile_groups=4),
         "tile_narrow": dict(tile_groups=2),
         "tile_narrow_res": dict(flags=gs.GS_SIM_TILE_DESC_RESIDENT),
         "tile_narrow_tma": dict(flags=gs.GS_SIM_TILE_DESC_TMA, tile_groups=2),
         "cluster_2": dict(cluster_size=2, slab_lanes=256),             # kernel C, DSMEM slab broadcast
         "cluster_8": dict(cluster_size=8, slab_lanes=256)}.get(kernel, {})
if kernel == "lut_u4":
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
for k in ${KERNELS:-lut poly ab tile lut_groups lut_u4 tile_tma tile_global tile_narrow tile_narrow_res tile_narrow_tma cluster_2 cluster_8}; do
  for tool in memcheck racecheck synccheck; do
    timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san_run.py $k > $OUT/${k}_${tool}.log 2>&1
    echo "$k $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $OUT/${k}_${tool}.log | tr '\n' ' ')" >> $OUT/summary.txt
  done
done
