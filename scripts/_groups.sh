O=gpurun_out/groups; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "lane_groups or bulk" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/rc.txt
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline "$@" 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); r=d.get('roofline') or {}; print('$*', '%.4g'%d['value'], '%.0f'%r.get('achieved',0), d['signature']['lane_sig_sum'])" >> $O/sweep.txt; }
for g in 1 2 4; do b --config C4 --lane-groups $g; done
for g in 1 2 4; do b --config C5 --lane-groups $g; done
for g in 1 2 4 8; do b --config C3 --lane-groups $g; done
for g in 1 2 4 8; do b --config C2 --kernel lut --lane-groups $g; done
