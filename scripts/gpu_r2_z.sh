#!/bin/bash
# descriptor L1 prefetch before the PDL wait: parity subset, then A/B vs the previous build
OUT=gpurun_out/${1:-r2z}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "multi_gate or slab or grid_stride or fuzz or c3 or c1" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
TAG=${1:-r2z} RUNS="--config C3;--config C4;--config C5 --steps 2;--config C5 --lane-groups 2 --slab-lanes 4096 --steps 2" VARIANTS="new head" bash scripts/ab_libs.sh
