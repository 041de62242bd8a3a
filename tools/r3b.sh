export BLU_GBY_JIT_VERBOSE=1
BLU_GBY_CSCATTER=1 timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 3 > gpurun_out/r3b_C3.json 2>gpurun_out/r3b_C3.err; echo rc=$?; python -c "
import json; d=json.load(open('gpurun_out/r3b_C3.json')); r=d['roofline']; print('C3 cs', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)}, d['config']['groups'])" || tail -5 gpurun_out/r3b_C3.err
BLU_GBY_CSCATTER=1 timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "partitioned or fanout or tma" > gpurun_out/r3b_tests.log 2>&1; grep -E "FAILED|Error" gpurun_out/r3b_tests.log | head -5; tail -1 gpurun_out/r3b_tests.log
