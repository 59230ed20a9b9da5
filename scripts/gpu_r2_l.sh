#!/bin/bash
OUT=gpurun_out/${1:-r2l}
mkdir -p $OUT
timeout 1500 python scripts/mid_size.py --gates 5000,10000,20000,40000 --flags 0,16,32 > $OUT/mid_size.jsonl 2> $OUT/mid_size.err; echo "mid rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/small.txt; }
for a in "--config C1 --kernel auto" "--config C2 --kernel auto" "--config C2 --kernel poly" "--config C4 --kernel poly --cycles-per-step 10" "--config C2 --kernel ab"; do b "$a"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -c 1 -o $OUT/prof_T \
  python bench.py --config C2 --kernel tile --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/ncu_T.log 2>&1; echo "ncu-T rc=$?" >> $OUT/rc.txt
