timeout 900 ncu --set full --clock-control none --import-source on -k regex:blu_jit_scatter -s 3 -c 1 -o gpurun_out/r2u_C5sc \
    python bench.py --config C5 --rows 400000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks > gpurun_out/r2u.out 2>&1; echo rc=$?
