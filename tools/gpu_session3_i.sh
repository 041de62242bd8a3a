# two-phase predicated shared-memory SUM updates: C2 / C4 (compare with r1d: C2 kernel 0.604 ms, C4 10.0 ms)
for c in C2 C4 C1; do
python bench.py --config $c --steps 20 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
done
python -m pytest tests/test_parity_gpu.py -x -q -k "config_parity or rank_front or forced_paths or small_and_ragged or i128 or wide" 2>&1 | tail -2
