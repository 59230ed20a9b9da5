#!/bin/bash
OUT=gpurun_out/${1:-r2t}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "tile or auto or c1 or c2 or fuzz or collapsed or degenerate" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/small.txt; }
for a in "--config C2 --kernel auto" "--config C1 --kernel auto"; do b "$a"; done
for G in 5000 10000; do timeout 300 python scripts/tile_mid_once.py --gates $G --flags 0 --cycles 50 >> $OUT/mid.jsonl 2>>$OUT/err.txt; done
KERNELS="tile_narrow tile_narrow_res tile_narrow_tma" timeout 2400 bash scripts/sanitize.sh r2t_san > $OUT/san.log 2>&1; echo "san rc=$?" >> $OUT/rc.txt
cp gpurun_out/r2t_san/summary.txt $OUT/san_summary.txt 2>/dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -c 1 -o $OUT/prof_T_C2 \
  python bench.py --config C2 --kernel tile --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/ncu_T.log 2>&1; echo "ncu-T rc=$?" >> $OUT/rc.txt
