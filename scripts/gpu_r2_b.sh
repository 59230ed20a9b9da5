#!/bin/bash
# round 2, call b: C4 full-size parity test, sub-batch size A/B on C5, in-situ traffic, kernel T profile
OUT=gpurun_out/${1:-r2b}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "c4_full or c5_every" > $OUT/pytest_c4c5.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
for s in 32768 65536; do
  timeout 600 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --sub-lanes $s > $OUT/bench_sub$s.json 2>>$OUT/bench.err; echo "bench sub $s rc=$?" >> $OUT/rc.txt
done
timeout 600 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_C4.json 2>>$OUT/bench.err; echo "bench C4 rc=$?" >> $OUT/rc.txt
timeout 600 python bench.py --config C2 --kernel tile --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_C2T.json 2>>$OUT/bench.err; echo "bench C2T rc=$?" >> $OUT/rc.txt
timeout 600 python bench.py --config C3 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_C3.json 2>>$OUT/bench.err; echo "bench C3 rc=$?" >> $OUT/rc.txt
timeout 900 python scripts/ncu_insitu.py --tag r02 -- --config C5 > $OUT/insitu_C5.log 2>&1; echo "insitu C5 rc=$?" >> $OUT/rc.txt
timeout 900 python scripts/ncu_insitu.py --tag r02 -- --config C4 > $OUT/insitu_C4.log 2>&1; echo "insitu C4 rc=$?" >> $OUT/rc.txt
cp profiles/traffic.json $OUT/traffic.json
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -s 1 -c 1 -o $OUT/prof_T \
  python bench.py --config C2 --kernel tile --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/ncu_T.log 2>&1; echo "ncu-T rc=$?" >> $OUT/rc.txt
