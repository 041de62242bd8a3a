# C4 rank-front profile (SASS-level) + host overhead of small executes
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"blu_jit_global" -s 2 -c 1 -o gpurun_out/s3c_prof_C4 env ITERS=3 python tools/phase_probe.py C4 > gpurun_out/s3c_prof_C4.log 2>&1
python tools/host_overhead.py C1 300 > gpurun_out/s3c_host_C1.txt 2>&1
python tools/host_overhead.py C2 100 > gpurun_out/s3c_host_C2.txt 2>&1
cat gpurun_out/s3c_host_C1.txt gpurun_out/s3c_host_C2.txt
