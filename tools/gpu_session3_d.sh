# C4: per-warp L2 prefetch of the next tile A/B
for i in 1 2; do
for E in BLU_GBY_AGG_PREFETCH=0 BLU_GBY_AGG_PREFETCH=1; do
env $E python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C4 $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3), r['kernel'])"
done; done
BLU_GBY_AGG_PREFETCH=1 python -m pytest tests/test_parity_gpu.py -x -q -k "rank_front or forced_paths or config_parity" 2>&1 | tail -2
