#!/bin/bash
# multi-gate warp units (kernel A on rows < 16,384 lanes): parity tests, C5 sub-batch-size A/B
# against a build without them (GS_LUT_GP=0, libgsim_nogp.so), in-situ DRAM bytes per cycle.
OUT=gpurun_out/${1:-r2u}
mkdir -p $OUT
P=paper_conf_ipps_gavierrprs23_b200
cp $P/libgsim.so $P/libgsim_new.so
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "multi_gate or grid_stride or fuzz" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 400 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $2 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1 $2', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['lane_groups'])" >> $OUT/sweep.txt; }
RUNS=("--config C5" "--config C5 --sub-lanes 16384" "--config C5 --sub-lanes 16384 --lane-groups 2" "--config C5 --sub-lanes 8192" "--config C5 --sub-lanes 8192 --lane-groups 1" "--config C5 --sub-lanes 4096" "--config C4" "--config C4 --lane-groups 8" "--config C4 --lane-groups 16")
for v in new nogp; do
  cp $P/libgsim_$v.so $P/libgsim.so
  for r in "${RUNS[@]}"; do b $v "$r"; done
done
cp $P/libgsim_new.so $P/libgsim.so
for r in "--config C5 --sub-lanes 8192" "--config C5 --sub-lanes 4096" "--config C5 --sub-lanes 16384"; do
  timeout 900 python scripts/ncu_insitu.py --tag r02u -- $r > $OUT/insitu_$(echo $r | tr ' ' '_').log 2>&1; echo "insitu $r rc=$?" >> $OUT/rc.txt
done
cp -r gpurun_out/insitu $OUT/ 2>/dev/null
cp profiles/traffic.json $OUT/traffic_u.json
