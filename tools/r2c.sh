mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_dist_gpu.py tests/test_bench_multirank_gpu.py -x -q > gpurun_out/r2c_dist.log 2>&1; tail -3 gpurun_out/r2c_dist.log
timeout 900 python bench.py > gpurun_out/r2c_bench.json 2> gpurun_out/r2c_bench.err; echo bench rc=$?; tail -c 600 gpurun_out/r2c_bench.json; tail -3 gpurun_out/r2c_bench.err
