# default two-level bucket-table mode for C3: full GPU suite + C3/C5 bench lines
python -m pytest tests -m gpu -x -q > gpurun_out/s3v_gputests.log 2>&1; tail -2 gpurun_out/s3v_gputests.log
for c in C3 C5; do
python bench.py --config $c --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', round(d['ms_per_step'],3), r['kernel'], round(r['frac'],3), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
done
