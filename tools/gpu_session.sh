#!/bin/bash
# One parameterised GPU-box session (run under gpurun): the GPU suite + smoke, the default bench line,
# and/or the launch list + ncu captures of the headline workload. Outputs land in gpurun_out/ with the
# TAG prefix (summarised into profiles/ by tools/ncu_summarize.py on the dev box).
#   TAG=r2x bash tools/gpu_session.sh [tests|bench|ncu|all] ...
# Per-config A/B timings: tools/ab_cfg.sh; the full per-config profile set: tools/capture_profiles.sh.
TAG=${TAG:-run}
O=gpurun_out; mkdir -p $O
for WHAT in "${@:-all}"; do
  if [ "$WHAT" = tests ] || [ "$WHAT" = all ]; then
    timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_gputests.log 2>&1; echo tests rc=$?; tail -2 $O/${TAG}_gputests.log
    timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo smoke rc=$?
  fi
  if [ "$WHAT" = bench ] || [ "$WHAT" = all ]; then
    timeout 900 python bench.py > $O/${TAG}_bench_default.json 2> $O/${TAG}_bench_default.err; echo bench rc=$?
  fi
  if [ "$WHAT" = ncu ] || [ "$WHAT" = all ]; then
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_default.csv \
        python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --sub '' > $O/${TAG}_launches_default.out 2>&1; echo launches rc=$?
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:blu_jit_scatter -s 3 -c 1 -o $O/${TAG}_prof_C5sc \
        python bench.py --config C5 --rows 400000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks > $O/${TAG}_prof_C5sc.out 2>&1; echo sc rc=$?
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:blu_jit_global -s 3 -c 1 -o $O/${TAG}_prof_C5p2 \
        python bench.py --config C5 --rows 400000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks > $O/${TAG}_prof_C5p2.out 2>&1; echo p2 rc=$?
  fi
done
