mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or partition or part" > gpurun_out/r2f_tests.log 2>&1; tail -1 gpurun_out/r2f_tests.log
for c in C3 C5; do
timeout 300 python bench.py --config $c --sub '' --no-e2e --no-cpu --steps 5 > gpurun_out/r2f_bench_$c.json 2>gpurun_out/r2f_bench_$c.err; echo rc=$?
python -c "
import json; d=json.load(open('gpurun_out/r2f_bench_$c.json')); r=d['roofline']; print('$c', round(d['ms_per_step'],2), r['kernel'], {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
done
BLU_GBY_PART_SMEM=1 timeout 300 python bench.py --config C5 --sub '' --no-e2e --no-cpu --steps 3 > gpurun_out/r2f_bench_C5smem.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r2f_bench_C5smem.json')); r=d['roofline']; print('C5 smem', round(d['ms_per_step'],2), d['config']['partitions'], {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
