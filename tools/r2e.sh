mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or partition or part" > gpurun_out/r2e_tests.log 2>&1; tail -2 gpurun_out/r2e_tests.log
timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 10 > gpurun_out/r2e_bench_C3.json 2>gpurun_out/r2e_bench_C3.err; echo rc=$?
python -c "
import json; d=json.load(open('gpurun_out/r2e_bench_C3.json')); r=d['roofline']; print('C3', d['ms_per_step'], r['kernel'], json.dumps(r['phases']))"
BLU_GBY_JIT_DUMP=/tmp timeout 600 ncu --set full --import-source on --clock-control none -k regex:blu_jit_global_3 -c 1 -o gpurun_out/r2e_C4 python bench.py --config C4 --rows 200000000 --sub '' --no-e2e --no-cpu --no-clocks --steps 1 --warmup 3 > gpurun_out/r2e_ncu_C4.log 2>&1; echo ncu rc=$?
