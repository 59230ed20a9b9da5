for u in 1 2 4; do for sl in 1 2 4 8; do
  timeout 120 python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu-baseline --lut-unroll $u --lane-slabs $sl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('U',$u,'slabs',$sl, 'value %.3e'%d['value'], 'ms/step %.1f'%d['ms_per_step'], 'lvl GB/s %.0f'%r['achieved'], 'share %.3f'%r['level_share_of_step'], 'lvl_us %.1f'%r['avg_level_launch_us'])"
done; done
