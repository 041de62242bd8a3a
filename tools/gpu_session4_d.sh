# session 4: 1 or 2 hot keys in registers — parity under HOT_REG=2, C4 A/B over CTA sizes
mkdir -p gpurun_out
O=gpurun_out/r1h_hotreg2.txt
: > $O
BLU_GBY_HOT_REG=2 python -m pytest tests -m gpu -q -x > gpurun_out/r1h_gputests_hotreg2.log 2>&1; tail -1 gpurun_out/r1h_gputests_hotreg2.log | tee -a $O
python -m pytest tests/test_parity_gpu.py -q -k "rank_front" >> $O 2>&1
for rep in 1 2; do
for cfg in "0 768" "1 640" "2 640" "2 576" "1 576"; do
  set -- $cfg
  echo "== HOT_REG=$1 BLOCK=$2 rep=$rep" >> $O
  BLU_GBY_HOT_REG=$1 BLU_GBY_BLOCK=$2 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu 2>>$O | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], r['avg_launch_ms'], r['kernel'], d['config']['block'], r['frac'])" >> $O 2>&1
done
done
cat $O
