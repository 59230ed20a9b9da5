O=gpurun_out/g3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "lane_groups or bulk or c4_full or c5_shard or launch_and_cache" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/rc.txt
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench rc=$?" >> $O/rc.txt
timeout 600 bash scripts/ncu_traffic_pass.sh C4; echo "tr4 rc=$?" >> $O/rc.txt
timeout 600 bash scripts/ncu_traffic_pass.sh C5; echo "tr5 rc=$?" >> $O/rc.txt
mv gpurun_out/traffic_C4.csv $O/traffic_C4_G4.csv; mv gpurun_out/traffic_C5.csv $O/traffic_C5_G2.csv
timeout 600 bash scripts/ncu_traffic_pass.sh C4 --lane-groups 1; mv gpurun_out/traffic_C4.csv $O/traffic_C4_G1.csv
cp gpurun_out/traffic_*.log $O/
