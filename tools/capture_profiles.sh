#!/bin/bash
# Run on the GPU box (gpurun): launch lists + ncu --set full of the dominant kernels, and bench lines.
# Outputs land in gpurun_out/ (summarised into profiles/ by tools/ncu_summarize.py on the dev box).
#   TAG=r1b bash tools/capture_profiles.sh [ncu|bench|all]
TAG=${TAG:-r1}
WHAT=${1:-all}
O=gpurun_out
if [ "$WHAT" = ncu ] || [ "$WHAT" = all ]; then
  # launch lists (cold-cache, serialised): the default bench command and C3
  ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $O/${TAG}_launches_C2.csv \
      python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${TAG}_launches_C3.csv \
      env ITERS=2 python tools/phase_probe.py C3 > /dev/null 2>&1
  # dominant kernels, one full capture each
  ncu --set full --clock-control none --import-source on -k regex:blu_jit_dense -s 3 -c 1 -o $O/${TAG}_prof_C2 \
      python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:blu_jit_dense -s 3 -c 1 -o $O/${TAG}_prof_C1 \
      python bench.py --config C1 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"blu_jit_global" -s 2 -c 1 -o $O/${TAG}_prof_C3p2 \
      env ITERS=3 python tools/phase_probe.py C3 > /dev/null 2>&1
  # C3's default two-level scatter: launch 0 = first level (input -> 32 buckets), launch 1 = one of the
  # 32 second-level launches (a bucket -> its 64 sub-buckets)
  ncu --set full --clock-control none --import-source on -k regex:"blu_jit_scatter" -s 0 -c 1 -o $O/${TAG}_prof_C3sc \
      env ITERS=1 python tools/phase_probe.py C3 > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"blu_jit_scatter" -s 1 -c 1 -o $O/${TAG}_prof_C3sc2 \
      env ITERS=1 python tools/phase_probe.py C3 > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"blu_jit_bucket" -s 0 -c 1 -o $O/${TAG}_prof_C3bk \
      env ITERS=1 python tools/phase_probe.py C3 > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"blu_jit_global" -s 2 -c 1 -o $O/${TAG}_prof_C4 \
      env ITERS=3 python tools/phase_probe.py C4 > /dev/null 2>&1
  # sort offload (NEXT-4): launch list and one radix downsweep (a level-2 pass: random digits)
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${TAG}_launches_S1.csv \
      python bench.py --config S1 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"k_rs_downsweep<unsigned long>" -s 6 -c 1 -o $O/${TAG}_prof_S1 \
      python bench.py --config S1 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"k_seg_warp_sort" -s 2 -c 1 -o $O/${TAG}_prof_S1w \
      python bench.py --config S1 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
fi
if [ "$WHAT" = bench ] || [ "$WHAT" = all ]; then
  python bench.py --steps 200 --warmup 5 > $O/${TAG}_bench_C2.json 2> $O/${TAG}_bench_C2.err
  for c in C1 C3 C4 C5; do
    python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > $O/${TAG}_bench_$c.json 2>> $O/${TAG}_bench_$c.err
  done
  python bench.py --config S1 --steps 10 --warmup 3 > $O/${TAG}_bench_S1.json 2> $O/${TAG}_bench_S1.err
  python bench.py --impl reference --steps 5 --warmup 3 > $O/${TAG}_bench_ref.json 2> $O/${TAG}_bench_ref.err
  python bench.py --impl reference --config S1 --steps 3 --warmup 1 > $O/${TAG}_bench_ref_S1.json 2> $O/${TAG}_bench_ref_S1.err
fi
