# N > 1 bench roofline bookkeeping (gloo, both ranks on cuda:0) + Python wrapper profile
export BLU_BENCH_DIST_BACKEND=gloo BLU_BENCH_DEVICE=0
R="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533"
for A in "" "--config C5 --rows 200000000" "--config C4 --rows 200000000"; do
timeout 600 $R bench.py --gpus 2 $A --steps 3 --warmup 3 --no-e2e 2> /dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print('$A', d['n_gpus'], round(d['ms_per_step'],3), d['config']['parallelism'], r['kernel'], round(r['avg_launch_ms'],4), round(r['frac'],3), r.get('phases') and {k:v for k,v in r['phases'].items() if k!='launches_per_step'})"
done
unset BLU_BENCH_DIST_BACKEND BLU_BENCH_DEVICE
python tools/py_profile.py 2>&1 | head -40
