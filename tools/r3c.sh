BLU_GBY_CSCATTER=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:blu_jit_cscatter -s 1 -c 1 -o gpurun_out/r3c_cs \
    python bench.py --config C3 --rows 200000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks > gpurun_out/r3c.out 2>&1; echo rc=$?
