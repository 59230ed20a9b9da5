O=gpurun_out/s4g; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'])" >> $O/sweep.txt; }
for a in "--config C3" "--config C3 --kernel tile --tile-slots-global" "--config C3 --kernel tile --tile-slots-global --tile-words 4 --tile-groups 1" "--config C3 --kernel tile --tile-slots-global --tile-words 4 --tile-groups 2" "--config C3 --kernel tile --tile-slots-global --tile-words 8 --tile-groups 1" "--config C4 --l2-hints 1" "--config C4"; do b "$a"; done
timeout 900 python scripts/mid_size.py --lanes 16384 --gates 20000,40000,100000 --flags 0,256 > $O/mid16k.txt 2>&1
timeout 900 python scripts/mid_size.py --lanes 65536 --gates 40000,100000 --flags 256 > $O/mid64k.txt 2>&1
