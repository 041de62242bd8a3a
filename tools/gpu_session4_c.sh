# session 4: hottest-key register accumulator (BLU_GBY_HOT_REG) — parity under the switch, C4 A/B
mkdir -p gpurun_out
O=gpurun_out/r1h_hotreg.txt
: > $O
BLU_GBY_HOT_REG=1 python -m pytest tests -m gpu -q -x > gpurun_out/r1h_gputests_hotreg.log 2>&1; tail -3 gpurun_out/r1h_gputests_hotreg.log | tee -a $O
for rep in 1 2; do
for hr in 0 1; do
  for blk in 768 640; do
    echo "== HOT_REG=$hr BLOCK=$blk rep=$rep" >> $O
    BLU_GBY_HOT_REG=$hr BLU_GBY_BLOCK=$blk python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu 2>>$O | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], r['avg_launch_ms'], r['kernel'], d['config']['block'], r['frac'])" >> $O 2>&1
  done
done
done
cat $O
