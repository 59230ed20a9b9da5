#!/bin/bash
# A/B of two builds of libgsim.so on ONE box (boxes differ by up to ~6 %): bench lines tagged
# new / head in gpurun_out/$TAG/sweep.txt, two repetitions each.  Prepare here:
#   git worktree add /tmp/headrepo <ref> && (cd /tmp/headrepo && python -m paper_conf_ipps_gavierrprs23_b200._build)
#   cp /tmp/headrepo/paper_conf_ipps_gavierrprs23_b200/libgsim.so paper_conf_ipps_gavierrprs23_b200/libgsim_head.so
# then: gpurun -- 'TAG=ab CONFIGS="C3 C4" bash scripts/ab_libs.sh'
O=gpurun_out/${TAG:-ab}; mkdir -p $O
P=paper_conf_ipps_gavierrprs23_b200
cp $P/libgsim.so $P/libgsim_new.so
b() { timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline "${@:2}" 2>>$O/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1 ${*:2}', '%.4g'%d['value'], d['signature']['lane_sig_sum'])" >> $O/sweep.txt; }
for rep in 1 2; do
 for v in new head; do
  cp $P/libgsim_$v.so $P/libgsim.so
  for c in ${CONFIGS:-C3 C4}; do b $v --config $c; done
 done
done
cp $P/libgsim_new.so $P/libgsim.so
