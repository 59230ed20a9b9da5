#!/bin/bash
OUT=gpurun_out/${1:-r2q}
mkdir -p $OUT
b() { timeout 900 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); r=d['roofline']; print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['lane_groups'], '%.3f'%r['frac'], r['avg_level_launch_us'])" >> $OUT/groups.txt; }
for a in "--config C4 --lane-groups 2" "--config C4 --lane-groups 4" "--config C4 --lane-groups 8" "--config C4 --lane-groups 1" "--config C5 --lane-groups 4" "--config C5 --lane-groups 1" "--config C4 --lut-unroll 2" "--config C5 --sub-lanes 65536 --lane-groups 4"; do b "$a"; done
echo done >> $OUT/rc.txt
