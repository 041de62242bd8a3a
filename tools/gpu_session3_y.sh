# register budget sweep: CTA size vs pipelined rows per thread (C4 front path, C2 dense path)
for E in "BLU_GBY_BLOCK=768 BLU_GBY_PIPE_R=4" "BLU_GBY_BLOCK=640 BLU_GBY_PIPE_R=4" "BLU_GBY_BLOCK=896 BLU_GBY_PIPE_R=4" "BLU_GBY_BLOCK=512 BLU_GBY_PIPE_R=4 BLU_GBY_JIT_MINB=1"; do
env $E python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C4 $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3))"
done
for E in "BLU_GBY_X=0" "BLU_GBY_BLOCK=768 BLU_GBY_CTAS_PER_SM=1 BLU_GBY_DENSE_PIPE_R=4" "BLU_GBY_BLOCK=1024 BLU_GBY_CTAS_PER_SM=1" "BLU_GBY_BLOCK=640 BLU_GBY_CTAS_PER_SM=1 BLU_GBY_DENSE_PIPE_R=4"; do
env $E python bench.py --config C2 --steps 30 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C2 $E', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3))"
done
