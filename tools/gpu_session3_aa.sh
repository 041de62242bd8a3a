# bucket-table pass 2 with double-buffered tile loads (768 x 80 regs) vs 1024 x 64 unpipelined
BLU_GBY_BUCKET_PIPE=1 python -m pytest tests/test_parity_gpu.py -x -q -k "partitioned" 2>&1 | tail -2
for E in "BLU_GBY_X=0" "BLU_GBY_BUCKET_PIPE=1" "BLU_GBY_BUCKET_PIPE=1 BLU_GBY_BUCKET_THREADS=512" "BLU_GBY_BUCKET_PIPE=1 BLU_GBY_BUCKET_THREADS=640"; do
env $E python bench.py --config C3 --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C3 $E', round(d['ms_per_step'],3), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
done
