#!/bin/bash
# kernel A slab schedule inside concurrent lane groups: parity tests, C5 sweep, in-situ DRAM
OUT=gpurun_out/${1:-r2x}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "slab or multi_gate" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/rc.txt
b() { timeout 400 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-roofline $1 2>>$OUT/err.txt | python -c "
import json,sys; d=json.load(sys.stdin); print('$1', '%.4g'%d['value'], d['signature']['lane_sig_sum'], d['clocks']['sm_mhz'], d['config']['lane_groups'], d['config']['launch']['slab_lanes'], d['gpu_launches'])" >> $OUT/sweep.txt; }
b "--config C5"
b "--config C5 --lane-groups 2 --slab-lanes 4096"
b "--config C5 --lane-groups 2 --slab-lanes 8192"
b "--config C5 --lane-groups 4 --slab-lanes 4096"
b "--config C5 --lane-groups 2 --slab-lanes 4096 --slab-min-gates 65536"
b "--config C5 --sub-lanes 65536 --lane-groups 2 --slab-lanes 8192"
b "--config C5 --sub-lanes 65536 --lane-groups 4 --slab-lanes 4096"
b "--config C5 --sub-lanes 65536 --lane-groups 2 --slab-lanes 4096"
b "--config C4 --lane-groups 4 --slab-lanes 8192"
b "--config C4 --lane-groups 2 --slab-lanes 8192"
for r in "--config C5 --lane-groups 2 --slab-lanes 4096" "--config C5 --lane-groups 2 --slab-lanes 8192"; do
  timeout 900 python scripts/ncu_insitu.py --tag r02x -- $r > $OUT/insitu_$(echo $r | tr ' ' '_').log 2>&1; echo "insitu $r rc=$?" >> $OUT/rc.txt
done
cp profiles/traffic.json $OUT/traffic_x.json
