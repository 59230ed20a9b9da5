#!/bin/bash
OUT=gpurun_out/${1:-r2m}
mkdir -p $OUT
for tw in 4 8 16 32; do for ng in 1 2 4; do
  timeout 600 python scripts/mid_size.py --gates 5000,10000 --flags 0,16,32 --tile-words $tw --tile-groups $ng > $OUT/mid_tw${tw}_ng${ng}.jsonl 2>> $OUT/err.txt
done; done
timeout 600 python scripts/mid_size.py --gates 5000,10000,20000 --flags 0 > $OUT/mid_auto.jsonl 2>> $OUT/err.txt
echo done >> $OUT/rc.txt
