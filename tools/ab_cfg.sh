#!/bin/bash
# A/B helper (run under gpurun): bench one config for each env assignment, alternating, twice each;
# prints step ms, dominant-kernel launch ms and its roofline fraction.
#   bash tools/ab_env.sh C4 "BLU_GBY_MMBOUND=0" "BLU_GBY_MMBOUND=1"
CFG=$1; shift
for i in 1 2; do
for E in "$@"; do
env $E timeout 600 python bench.py --config $CFG --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks --sub '' 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$CFG $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3), r['kernel'])"
done; done
