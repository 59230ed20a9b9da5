#!/bin/bash
# kernel T configs on C2 with ALAP levels (256 live slots); kernel C first light on C3/C4
OUT=gpurun_out/${1:-r2d}
mkdir -p $OUT
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'])" >> $OUT/sweep.txt; }
for a in "--config C2 --kernel tile" "--config C2 --kernel tile --tile-words 64 --tile-groups 1" "--config C2 --kernel tile --tile-words 64 --tile-groups 2" \
  "--config C2 --kernel tile --tile-words 32 --tile-groups 4" "--config C2 --kernel tile --tile-words 32 --tile-groups 2" "--config C2 --kernel tile --tile-words 32 --tile-groups 1" \
  "--config C2 --kernel tile --tile-words 64 --tile-groups 1 --tile-desc tma" "--config C2 --kernel lut" "--config C1 --kernel tile"; do b "$a"; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tile or c2 or fuzz" > $OUT/pytest_tile.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
for a in "--config C3 --kernel cluster --cycles-per-step 20" "--config C3" ; do b "$a"; done
