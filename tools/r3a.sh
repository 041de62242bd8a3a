timeout 900 python -m pytest tests/test_dist_gpu.py tests/test_bench_multirank_gpu.py -q -x 2>&1 | tail -1
