# A/B helper: C2 bench (kernel time + frac) for each env assignment given as arguments, twice.
for i in 1 2; do
for E in "$@"; do
env $E python bench.py --steps 200 --warmup 5 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$E', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
done; done
