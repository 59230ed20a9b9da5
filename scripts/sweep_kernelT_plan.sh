#!/bin/bash
# kernel T plan sweep (tile words x thread groups) on C2 vs the chooser's pick
O=gpurun_out/${TAG:-s4tp}; mkdir -p $O
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'])" >> $O/sweep.txt; }
for tw in "" "--tile-words 64 --tile-groups 1" "--tile-words 32 --tile-groups 1" "--tile-words 32 --tile-groups 2" "--tile-words 16 --tile-groups 2" "--tile-words 16 --tile-groups 4" "--tile-words 8 --tile-groups 4"; do
  b "--config C2 --kernel tile $tw"
done
