# host-side launch path: JIT handle cache + deferred output allocation (r1d: C2 step 0.678 ms, c_call 752 us)
python tools/host_overhead.py C1 300; python tools/host_overhead.py C2 100
for c in C2 C1 C4; do
python bench.py --config $c --steps 30 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3))"
done
python -m pytest tests/test_parity_gpu.py -x -q 2>&1 | tail -2
