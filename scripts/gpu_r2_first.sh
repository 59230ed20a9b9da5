#!/bin/bash
# round-2 first validation call: host info, smoke, default bench (C5), GPU tests with timings
OUT=gpurun_out/${1:-r2a}
mkdir -p $OUT
(nproc; lscpu | head -20; nvidia-smi; free -g) > $OUT/host.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/rc.txt
timeout 1500 python bench.py --steps 3 --warmup 3 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/rc.txt
timeout 2400 python -m pytest tests -m gpu -q --durations=40 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
