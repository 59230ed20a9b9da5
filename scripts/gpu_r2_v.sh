#!/bin/bash
# multi-gate warp units: occupancy / gates-per-unit variants on small C5 sub-batches, per-level
# ncu of one 4,096-lane cycle (warm L2: --cache-control none), full capture of two big launches.
OUT=gpurun_out/${1:-r2v}
mkdir -p $OUT
P=paper_conf_ipps_gavierrprs23_b200
cp $P/libgsim.so $P/libgsim_new.so
b() { timeout 400 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $2 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1 $2', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['lane_groups'])" >> $OUT/sweep.txt; }
RUNS=("--config C5 --sub-lanes 4096" "--config C5 --sub-lanes 8192")
for v in new m2 m4 v8; do
  cp $P/libgsim_$v.so $P/libgsim.so
  for r in "${RUNS[@]}"; do b $v "$r"; done
done
cp $P/libgsim_new.so $P/libgsim.so
b new "--config C5"
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,lts__t_sector_hit_rate.pct,launch__grid_size"
timeout 900 ncu --cache-control none --clock-control none --metrics $M -s 240 -c 110 --csv --log-file $OUT/levels_4096.csv \
  python bench.py --config C5 --sub-lanes 4096 --quick --steps 1 --warmup 1 --cycles-per-step 3 > $OUT/ncu_levels.log 2>&1; echo "ncu-levels rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_level_lut_gp -s 300 -c 2 -o $OUT/prof_GP_4096 \
  python bench.py --config C5 --sub-lanes 4096 --quick --steps 1 --warmup 1 --cycles-per-step 3 > $OUT/ncu_full.log 2>&1; echo "ncu-full rc=$?" >> $OUT/rc.txt
