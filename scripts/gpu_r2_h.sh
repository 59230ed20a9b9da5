#!/bin/bash
OUT=gpurun_out/${1:-r2h}
mkdir -p $OUT
b() { timeout 900 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); r=d['roofline']; print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['levels'], '%.3f'%r['frac'])" >> $OUT/levels_ab.txt; }
for a in "--config C4 --levels balanced" "--config C4 --levels asap" "--config C4 --levels alap" "--config C5 --levels balanced" "--config C5 --levels asap" "--config C5 --levels alap" "--config C3 --levels alap"; do b "$a"; done
c() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/tile.txt; }
for a in "--tile-words 64 --tile-groups 2 --tile-desc global" "--tile-words 32 --tile-groups 4 --tile-desc global" "--tile-words 64 --tile-groups 2" "--tile-words 64 --tile-groups 1"; do c "--config C2 --kernel tile $a"; done
