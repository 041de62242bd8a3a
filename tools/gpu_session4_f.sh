# session 4: CTA size sweep around 640 threads with the hottest key in registers (C4)
mkdir -p gpurun_out
O=gpurun_out/r1i_block_sweep.txt
: > $O
for rep in 1 2; do
for blk in 640 672 704 608; do
  echo "== HOT_REG=1 BLOCK=$blk rep=$rep" >> $O
  BLU_GBY_BLOCK=$blk python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu 2>>$O | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], r['avg_launch_ms'], r['kernel'], d['config']['block'], r['frac'])" >> $O 2>&1
done
done
cat $O
