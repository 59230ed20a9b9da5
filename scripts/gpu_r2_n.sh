#!/bin/bash
OUT=gpurun_out/${1:-r2n}
mkdir -p $OUT
for f in 512 16; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tile -s 1 -c 1 -o $OUT/prof_5k_f$f \
  python scripts/tile_mid_once.py --gates 5000 --flags $f --tw 16 --ng 1 > $OUT/ncu_$f.log 2>&1; echo "ncu $f rc=$?" >> $OUT/rc.txt
done
timeout 600 python scripts/mid_size.py --gates 5000,10000 --flags 0 > $OUT/mid_auto.jsonl 2>> $OUT/err.txt
