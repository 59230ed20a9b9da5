O=gpurun_out/s4sw; mkdir -p $O
b() { timeout 400 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['config']['lane_groups'])" >> $O/sweep.txt; }
for c in C4 C3; do
 for a in "" "--lane-groups 2" "--lane-groups 8" "--lane-groups 1" "--lut-unroll 8" ; do b "--config $c $a"; done
done
for a in "" "--lane-groups 4" "--lane-groups 1"; do b "--config C5 --lanes 32768 $a"; done
