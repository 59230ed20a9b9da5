O=gpurun_out/gp; mkdir -p $O
for a in "--config C4" "--config C4 --lane-groups 1" "--config C5" "--config C3"; do
  n=$(echo $a | tr -d ' -')
  timeout 600 ncu --graph-profiling graph --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -c 4 --csv --log-file $O/$n.csv python bench.py $a --quick --steps 1 --warmup 1 --cycles-per-step 2 > $O/$n.log 2>&1
done
