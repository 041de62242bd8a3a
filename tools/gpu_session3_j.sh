# one branch per row in the JIT apply paths: C2 / C4 / C3 (r1d: C2 kernel 0.604 ms, C4 10.0 ms, C3 pass2 25.9 ms)
for c in C2 C4; do
python bench.py --config $c --steps 20 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
done
python bench.py --config C3 --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C3', round(d['ms_per_step'],3), r['phases']['scatter']['avg_launch_ms'], r['phases']['pass2']['avg_launch_ms'])"
python -m pytest tests/test_parity_gpu.py -x -q -k "config_parity or rank_front or forced_paths or small_and_ragged or key_range or wide or partition" 2>&1 | tail -2
