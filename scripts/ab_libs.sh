#!/bin/bash
# A/B of builds of libgsim.so on ONE box (boxes differ by up to ~6 %): bench lines tagged by
# variant in gpurun_out/$TAG/sweep.txt, two repetitions each.  Prepare here:
#   git worktree add /tmp/headrepo <ref> && (cd /tmp/headrepo && python -m paper_conf_ipps_gavierrprs23_b200._build)
#   cp /tmp/headrepo/paper_conf_ipps_gavierrprs23_b200/libgsim.so paper_conf_ipps_gavierrprs23_b200/libgsim_head.so
#   (further variants: GS_NVCC_EXTRA="-D..." python -m paper_conf_ipps_gavierrprs23_b200._build --force,
#    then copy libgsim.so to libgsim_<name>.so and list <name> in VARIANTS)
# then: gpurun -- 'TAG=ab RUNS="--config C3;--config C2 --kernel tile" VARIANTS="new head" bash scripts/ab_libs.sh'
O=gpurun_out/${TAG:-ab}; mkdir -p $O
P=paper_conf_ipps_gavierrprs23_b200
[ -f $P/libgsim_new.so ] || cp $P/libgsim.so $P/libgsim_new.so
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $2 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1 $2', '%.4g'%d['value'], d['signature']['lane_sig_sum'])" >> $O/sweep.txt; }
IFS=';' read -ra R <<< "${RUNS:---config C3;--config C4}"
for rep in 1 2; do
 for v in ${VARIANTS:-new head}; do
  cp $P/libgsim_$v.so $P/libgsim.so
  for r in "${R[@]}"; do b $v "$r"; done
 done
done
cp $P/libgsim_new.so $P/libgsim.so
