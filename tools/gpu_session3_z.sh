# 768-thread front CTAs with 4 pipelined rows per thread (default now): parity + C4 bench
python -m pytest tests/test_parity_gpu.py tests/test_fullsize_gpu.py -x -q -k "rank_front or forced_paths or key_range or config_parity or c4" 2>&1 | tail -2
python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C4', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3), r['kernel'], d['config']['block'])"
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
