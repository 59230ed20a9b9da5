#!/bin/bash
OUT=gpurun_out/${1:-r2e}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "cluster or tile or fuzz" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/sweep.txt; }
for a in "--config C2 --kernel tile" "--config C3 --kernel cluster --cycles-per-step 20" "--config C3 --kernel cluster --cycles-per-step 20 --cluster-size 1 --slab-lanes 128" "--config C3 --kernel cluster --cycles-per-step 20 --cluster-size 4 --slab-lanes 512"; do b "$a"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_cluster -c 1 -o $OUT/prof_C \
  python bench.py --config C3 --kernel cluster --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/ncu_C.log 2>&1; echo "ncu-C rc=$?" >> $OUT/rc.txt
