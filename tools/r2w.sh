timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "host" > gpurun_out/r2w_tests.log 2>&1; tail -1 gpurun_out/r2w_tests.log
timeout 900 python bench.py --sub '' --no-cpu > gpurun_out/r2w_bench.json 2>gpurun_out/r2w_bench.err; python -c "
import json; d=json.load(open('gpurun_out/r2w_bench.json')); print(round(d['ms_per_step'],2), d['e2e'])"
