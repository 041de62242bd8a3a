# C4: 768-thread CTAs (80 registers) with 2 or 4 pipelined rows per thread vs the default 1024 x 2
for i in 1 2; do
for E in "BLU_GBY_X=0" "BLU_GBY_BLOCK=768" "BLU_GBY_BLOCK=768 BLU_GBY_PIPE_R=4"; do
env $E python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C4 $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3), r['kernel'])"
done; done
