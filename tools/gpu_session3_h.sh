# sort downsweep pipelining (S1) + new defaults on C3 + sort parity
python bench.py --config S1 --steps 5 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('S1', round(d['ms_per_step'],3), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
python bench.py --config C3 --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C3', round(d['ms_per_step'],3), r['phases']['scatter']['avg_launch_ms'], r['phases']['pass2']['avg_launch_ms'])"
python -m pytest tests/test_sort_gpu.py -x -q 2>&1 | tail -2
