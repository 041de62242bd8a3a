set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m pytest tests -m gpu -x -q > gpurun_out/s3_gputests.log 2>&1; tail -3 gpurun_out/s3_gputests.log
python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/s3_C4.json 2>gpurun_out/s3_C4.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"blu_jit_global" -s 2 -c 1 -o gpurun_out/s3_prof_C4 env ITERS=3 python tools/phase_probe.py C4 > gpurun_out/s3_prof_C4.log 2>&1
ls -la gpurun_out
