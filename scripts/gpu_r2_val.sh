#!/bin/bash
# full validation: smoke, all GPU tests, default bench (C5), in-situ traffic of the benched
# build/program (C5, C4), ncu launch list of the default bench, ncu --set full of kernel A on C5
OUT=gpurun_out/${1:-r2val}
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/rc.txt
timeout 2400 python -m pytest tests -m gpu -q --durations=30 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
timeout 1500 python bench.py --steps 5 --warmup 3 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/rc.txt
timeout 900 python scripts/ncu_insitu.py --tag r02 -- --config C5 > $OUT/insitu_C5.log 2>&1; echo "insitu C5 rc=$?" >> $OUT/rc.txt
timeout 900 python scripts/ncu_insitu.py --tag r02 -- --config C4 > $OUT/insitu_C4.log 2>&1; echo "insitu C4 rc=$?" >> $OUT/rc.txt
cp profiles/traffic.json $OUT/traffic.json; cp profiles/r02_insitu_* $OUT/ 2>/dev/null
timeout 900 python bench.py --config C4 --steps 10 --warmup 3 > $OUT/bench_C4.json 2> $OUT/bench_C4.err; echo "bench C4 rc=$?" >> $OUT/rc.txt
timeout 900 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_C5_roof.json 2>> $OUT/bench.err; echo "bench C5 roof rc=$?" >> $OUT/rc.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1500 --csv --log-file $OUT/launches.csv \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_launch.log 2>&1; echo "ncu-launch rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_level_lut_wide -s 300 -c 3 -o $OUT/prof_A_C5 \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_A.log 2>&1; echo "ncu-A rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['launch'])" >> $OUT/small.txt; }
for a in "--config C1 --kernel tile" "--config C1 --kernel tile --tile-words 4 --tile-groups 1" "--config C1 --kernel tile --tile-words 32 --tile-groups 1" "--config C1 --kernel auto" "--config C2 --kernel tile" "--config C2 --kernel auto" "--config C3"; do b "$a"; done
