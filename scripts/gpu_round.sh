#!/bin/bash
# One gpurun call: smoke, GPU parity tests, default bench, ncu launch list, ncu full capture.
# Usage (from the repo root, under gpurun):  bash scripts/gpu_round.sh <tag>
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/rc.txt
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/rc.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $OUT/launches.csv \
  python bench.py --quick --steps 2 --warmup 1 --cycles-per-step 2 > $OUT/ncu_launch.log 2>&1; echo "ncu-launch rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_level_lut -s ${NCU_SKIP:-100} -c 3 -o $OUT/prof \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_full.log 2>&1; echo "ncu-full rc=$?" >> $OUT/rc.txt
