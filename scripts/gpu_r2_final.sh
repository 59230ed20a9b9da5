#!/bin/bash
# round-2 final validation on the frozen build: smoke, every GPU test, in-situ traffic of the
# benched build/program, the default bench as the driver runs it, C4, the reference arm, a
# 2-rank run on one device (gloo; the strong-scaled sharding path), ncu launch list and full
# captures of kernels A (C5) and T (C2), the small configs.
OUT=gpurun_out/${1:-r2final}
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/rc.txt
timeout 2400 python -m pytest tests -m gpu -q --durations=20 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
timeout 900 python scripts/ncu_insitu.py --tag r02 -- --config C5 > $OUT/insitu_C5.log 2>&1; echo "insitu C5 rc=$?" >> $OUT/rc.txt
timeout 900 python scripts/ncu_insitu.py --tag r02 -- --config C4 > $OUT/insitu_C4.log 2>&1; echo "insitu C4 rc=$?" >> $OUT/rc.txt
cp profiles/traffic.json $OUT/traffic.json; cp profiles/r02_insitu_* $OUT/ 2>/dev/null
timeout 2400 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/rc.txt
timeout 1200 python bench.py --config C4 --steps 10 --warmup 3 > $OUT/bench_C4.json 2> $OUT/bench_C4.err; echo "bench C4 rc=$?" >> $OUT/rc.txt
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_ref.json 2> $OUT/bench_ref.err; echo "bench ref rc=$?" >> $OUT/rc.txt
timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py \
  --gpus 2 --steps 1 --warmup 3 --dist-backend gloo --same-device --no-cpu-baseline --no-e2e > $OUT/bench_2rank_same_device.json 2> $OUT/bench_2rank.err; echo "bench 2rank rc=$?" >> $OUT/rc.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1500 --csv --log-file $OUT/launches.csv \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_launch.log 2>&1; echo "ncu-launch rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_level_lut_wide -s 300 -c 3 -o $OUT/prof_A_C5 \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_A.log 2>&1; echo "ncu-A rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -c 1 -o $OUT/prof_T_C2 \
  python bench.py --config C2 --kernel tile --quick --steps 1 --warmup 1 --cycles-per-step 4 > $OUT/ncu_T.log 2>&1; echo "ncu-T rc=$?" >> $OUT/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline $1 2>>$OUT/err.txt > $OUT/small_$2.json; echo "small $2 rc=$?" >> $OUT/rc.txt; }
b "--config C1 --kernel auto" C1; b "--config C2 --kernel auto" C2; b "--config C3" C3
