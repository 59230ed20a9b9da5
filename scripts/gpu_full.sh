#!/bin/bash
# Full validation + measurement pass (one gpurun call): GPU tests, smoke, default bench,
# ncu launch list of the bench, ncu --set full of kernel A (C4, steady-state cycle) and
# kernel T (C2), per-cycle level traffic (kernel-serialised) and in-situ graph traffic.
TAG=${1:-full}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/rc.txt
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/rc.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file $OUT/launches.csv \
  python bench.py --quick --steps 2 --warmup 1 --cycles-per-step 2 > $OUT/ncu_launch.log 2>&1; echo "ncu-launch rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_level_lut_wide -s ${NCU_SKIP:-280} -c 3 -o $OUT/prof_A \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_A.log 2>&1; echo "ncu-A rc=$?" >> $OUT/rc.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -s 1 -c 1 -o $OUT/prof_T \
  python bench.py --config C2 --kernel tile --quick --steps 1 --warmup 1 --cycles-per-step 2 > $OUT/ncu_T.log 2>&1; echo "ncu-T rc=$?" >> $OUT/rc.txt
timeout 600 bash scripts/ncu_traffic_pass.sh C4; mv gpurun_out/traffic_C4.csv $OUT/traffic_cycle_C4.csv; echo "traffic rc=$?" >> $OUT/rc.txt
timeout 600 ncu --graph-profiling graph --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
  --clock-control none -c 4 --csv --log-file $OUT/graph_C4.csv python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 \
  > $OUT/graph_C4.log 2>&1; echo "graph rc=$?" >> $OUT/rc.txt
