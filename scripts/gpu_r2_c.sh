#!/bin/bash
# kernel T v2: tests, C2/C1/mid-size configs, ncu
OUT=gpurun_out/${1:-r2c}
mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "tile or fuzz or aes or auto or degenerate or stimulus_hash or sub_batches or streamed or collapsed or wide" > $OUT/pytest_tile.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'])" >> $OUT/sweep.txt; }
for a in "--config C2 --kernel tile" "--config C2 --kernel tile --tile-words 64 --tile-groups 1 --tile-desc tma" "--config C2 --kernel tile --tile-words 32 --tile-groups 2" "--config C2 --kernel tile --tile-words 16 --tile-groups 4" "--config C2 --kernel tile --tile-words 64 --tile-groups 1" "--config C2 --kernel lut" "--config C1 --kernel tile" "--config C1 --kernel lut"; do b "$a"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -s 1 -c 1 -o $OUT/prof_T \
  python bench.py --config C2 --kernel tile --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/ncu_T.log 2>&1; echo "ncu-T rc=$?" >> $OUT/rc.txt
