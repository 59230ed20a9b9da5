#!/bin/bash
OUT=gpurun_out/${1:-r2o}
mkdir -p $OUT
for rep in 1 2; do
for G in 5000 10000; do for f in 0 512 16 32; do for cfg in "--tw 0 --ng 0" "--tw 16 --ng 1" "--tw 8 --ng 2" "--tw 8 --ng 1" "--tw 4 --ng 4"; do
  timeout 300 python scripts/tile_mid_once.py --gates $G --flags $f --cycles 50 $cfg >> $OUT/mid_fresh.jsonl 2>>$OUT/err.txt
done; done; done; done
echo done >> $OUT/rc.txt
