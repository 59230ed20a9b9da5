O=gpurun_out/groups2; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline "$@" 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); r=d.get('roofline') or {}; print('$*', '%.4g'%d['value'], '%.0f'%r.get('achieved',0), d['gpu_launches'], d['signature']['lane_sig_sum'])" >> $O/sweep.txt; }
b --config C4
b --config C4 --lane-groups 8
b --config C4 --lane-groups 4
b --config C5
b --config C3
b --config C2 --kernel lut
b --config C2 --kernel lut --lane-groups 2
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_level_lut_wide -s 200 -c 4 -o $O/prof_C4g4 \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 > $O/ncu_C4.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file $O/launches.csv \
  python bench.py --quick --steps 2 --warmup 1 --cycles-per-step 2 > $O/ncu_launch.log 2>&1
