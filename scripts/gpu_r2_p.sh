#!/bin/bash
OUT=gpurun_out/${1:-r2p}
mkdir -p $OUT
for G in 5000 10000; do for f in 512 16 32; do for cfg in "--tw 16 --ng 1" "--tw 8 --ng 2" "--tw 8 --ng 1"; do
  timeout 300 python scripts/tile_mid_once.py --gates $G --flags $f --cycles 50 $cfg >> $OUT/mid_fresh.jsonl 2>>$OUT/err.txt
done; done; done
for G in 5000 10000 20000; do timeout 300 python scripts/tile_mid_once.py --gates $G --flags 0 --cycles 50 >> $OUT/mid_fresh.jsonl 2>>$OUT/err.txt; done
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/c2.txt; }
for a in "--tile-desc resident --tile-words 64 --tile-groups 1" "--tile-desc global --tile-words 64 --tile-groups 1" "--tile-desc global --tile-words 64 --tile-groups 2" "--tile-desc tma --tile-words 64 --tile-groups 2" "--tile-desc resident --tile-words 32 --tile-groups 2"; do b "--config C2 --kernel tile $a"; done
echo done >> $OUT/rc.txt
