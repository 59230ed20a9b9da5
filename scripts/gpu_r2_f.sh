#!/bin/bash
OUT=gpurun_out/${1:-r2f}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "cluster" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch']['grid'])" >> $OUT/sweep.txt; }
for a in "--cluster-size 1 --slab-lanes 128" "--cluster-size 2 --slab-lanes 128" "--cluster-size 2 --slab-lanes 256" "--cluster-size 4 --slab-lanes 512" "--cluster-size 8 --slab-lanes 1024" "--cluster-size 4 --slab-lanes 256"; do b "--config C3 --kernel cluster --cycles-per-step 20 $a"; done
for a in "--cluster-size 2 --slab-lanes 256" "--cluster-size 4 --slab-lanes 512" "--cluster-size 8 --slab-lanes 1024"; do b "--config C4 --kernel cluster --cycles-per-step 10 $a"; done
