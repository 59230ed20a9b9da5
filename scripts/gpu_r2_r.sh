#!/bin/bash
OUT=gpurun_out/${1:-r2r}
mkdir -p $OUT
b() { timeout 1200 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); r=d['roofline']; print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['lane_groups'], '%.3f'%r['frac'], r['avg_level_launch_us'])" >> $OUT/sub.txt; }
for a in "--sub-lanes 16384" "--sub-lanes 16384 --lane-groups 1" "--sub-lanes 8192" "--sub-lanes 8192 --lane-groups 1" "--sub-lanes 4096"; do b "--config C5 $a"; done
for a in "--sub-lanes 8192" "--sub-lanes 4096"; do
  timeout 900 python scripts/ncu_insitu.py --tag r02slab -- --config C5 $a > $OUT/insitu_$(echo $a | tr -d ' -').log 2>&1
done
cp profiles/traffic.json $OUT/traffic.json
echo done >> $OUT/rc.txt
