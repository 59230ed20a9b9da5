#!/bin/bash
OUT=gpurun_out/${1:-r2s}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "tile or auto or c1 or c2 or fuzz or aes or collapsed or degenerate or streamed or stimulus_hash or sub_batches" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/small.txt; }
for a in "--config C2 --kernel auto" "--config C2 --kernel tile --tile-desc resident --tile-words 64 --tile-groups 2" "--config C2 --kernel tile --tile-desc global --tile-words 64 --tile-groups 2" "--config C2 --kernel tile --tile-desc tma --tile-words 64 --tile-groups 2" "--config C2 --kernel tile --tile-desc resident --tile-words 32 --tile-groups 4" "--config C1 --kernel auto"; do b "$a"; done
KERNELS="tile tile_tma tile_global" timeout 2400 bash scripts/sanitize.sh r2s_san > $OUT/san.log 2>&1; echo "san rc=$?" >> $OUT/rc.txt
cp gpurun_out/r2s_san/summary.txt $OUT/san_summary.txt 2>/dev/null
