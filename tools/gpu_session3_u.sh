# two-level scatter for the shared-memory bucket tables (C3, C5) vs the default L2-slice mode
python -m pytest tests/test_parity_gpu.py -x -q -k "partitioned" 2>&1 | tail -2
for E in "BLU_GBY_X=0" "BLU_GBY_PART_SMEM=1 BLU_GBY_PART_2LEVEL=1" "BLU_GBY_PART_SMEM=1"; do
env $E python bench.py --config C3 --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C3 $E', round(d['ms_per_step'],3), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
done
for E in "BLU_GBY_X=0" "BLU_GBY_PART_SMEM=1 BLU_GBY_PART_2LEVEL=1"; do
env $E python bench.py --config C5 --steps 3 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C5 $E', round(d['ms_per_step'],3), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
done
