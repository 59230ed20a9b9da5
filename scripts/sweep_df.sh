#!/bin/bash
# Kernel D parameter sweep on C4 (one gpurun call) + ncu captures of kernel D and of kernel A
# with lane slabs (L2 hit rates).  usage: bash scripts/sweep_df.sh <tag> [extra bench args]
OUT=gpurun_out/${1:-df_sweep}
mkdir -p $OUT
run() {
  timeout 300 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline "$@" 2>>$OUT/err.txt | python -c "import json,sys
for l in sys.stdin:
  l=l.strip()
  if not l.startswith('{'): continue
  d=json.loads(l); r=d['roofline']
  print('$*'.ljust(55), 'value %.3e'%d['value'], 'ms/step %.1f'%d['ms_per_step'], 'lvl GB/s %.0f'%r['achieved'], 'frac %.3f'%r['frac'], 'share %.3f'%r['level_share_of_step'])" >> $OUT/sweep.txt
}
if [ -n "$SWEEP" ]; then
  for a in $SWEEP; do run ${a//,/ }; done
else
run --kernel lut
for I in 2 4 8; do for G in 4 8 16; do run --kernel df --df-interleave $I --df-gpw $G; done; done
run --kernel df --lane-slabs 8 --df-interleave 4
run --kernel df --lane-slabs 4 --df-interleave 2
fi
if [ -n "$NCU" ]; then
timeout 600 ncu --set full --clock-control none -k regex:k_dataflow -s 2 -c 1 -o $OUT/prof_df \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 --kernel df --df-interleave 4 > $OUT/ncu_df.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:k_level_lut -s 300 -c 2 -o $OUT/prof_slab8 \
  python bench.py --quick --steps 1 --warmup 1 --cycles-per-step 2 --lane-slabs 8 > $OUT/ncu_slab8.log 2>&1
fi
