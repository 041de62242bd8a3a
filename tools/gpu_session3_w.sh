# C5 with 16384 bucket tables behind the two-level scatter (default now) vs the L2-slice mode
python -m pytest tests/test_parity_gpu.py -x -q -k "partitioned or C5 or regrow" 2>&1 | tail -2
for E in "BLU_GBY_X=0" "BLU_GBY_PART_SMEM=0"; do
env $E python bench.py --config C5 --steps 3 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C5 $E', round(d['ms_per_step'],3), r['kernel'], round(r['frac'],3), d['config']['partitions'], {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)}, r['phases']['launches_per_step'])"
done
python -m pytest tests/test_fullsize_gpu.py -x -q -k "c5 or c3" 2>&1 | tail -2
