#!/bin/bash
OUT=gpurun_out/${1:-r2g}
mkdir -p $OUT
timeout 1500 python scripts/ncu_level_issue.py --tag r02 --config C4 C3 > $OUT/level_issue.log 2>&1; echo "level-issue rc=$?" >> $OUT/rc.txt
cp profiles/r02_level_issue_* $OUT/ 2>/dev/null
b() { timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); r=d['roofline']; print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['levels'], '%.3f'%r['frac'], '%.1f'%r['avg_level_launch_us'])" >> $OUT/balance_ab.txt; }
for rep in 1 2; do for a in "--config C4" "--config C4 --no-balance" "--config C3" "--config C3 --no-balance"; do b "$a"; done; done
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_cluster -c 1 --csv --log-file $OUT/kernelC_C4_dram.csv \
  python bench.py --config C4 --kernel cluster --cluster-size 8 --slab-lanes 1024 --quick --steps 1 --warmup 1 --cycles-per-step 10 > $OUT/kc.log 2>&1; echo "kc rc=$?" >> $OUT/rc.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_cluster -c 1 -o $OUT/prof_C3_cs8 \
  python bench.py --config C3 --kernel cluster --cluster-size 8 --slab-lanes 1024 --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/kc3.log 2>&1; echo "kc3 rc=$?" >> $OUT/rc.txt
