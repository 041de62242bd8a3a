# Round-2 profiles of the headline workload (C5) and the default bench line. Run under gpurun.
O=gpurun_out; mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r2_launches_default.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --sub '' > $O/r2_launches_default.out 2>&1; echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:blu_jit_scatter -s 3 -c 1 -o $O/r2_prof_C5sc \
    python bench.py --config C5 --rows 400000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks > $O/r2_prof_C5sc.out 2>&1; echo sc rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:blu_jit_global_2_4_0_0_2 -s 3 -c 1 -o $O/r2_prof_C5p2 \
    python bench.py --config C5 --rows 400000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks > $O/r2_prof_C5p2.out 2>&1; echo p2 rc=$?
timeout 900 python bench.py > $O/r2_bench_default.json 2> $O/r2_bench_default.err; echo bench rc=$?
