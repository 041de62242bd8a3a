# A/B helper: bench one config (arg 1) for each env assignment (remaining args), twice each.
CFG=$1; shift
for i in 1 2; do
for E in "$@"; do
env $E python bench.py --config $CFG --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$CFG $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3), r['kernel'])"
done; done
