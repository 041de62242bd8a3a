#!/bin/bash
# One ncu --set full capture per dominant kernel of each config (run under gpurun, one GPU), for the
# round's profiles/ summaries (tools/ncu_summarize.py). TAG names the round.
TAG=${TAG:-r2f}
O=gpurun_out
B="python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e --no-clocks --sub ''"
cap() {  # name kernel-regex skip config rows
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$2 -s $3 -c 1 -o $O/${TAG}_prof_$1 \
    python bench.py --config $4 ${5:+--rows $5} --steps 1 --warmup 1 --no-cpu --no-e2e --no-clocks --sub '' > $O/${TAG}_prof_$1.out 2>&1
  echo "$1 rc=$?"
}
cap C2 blu_jit_dense 1 C2
cap C1 blu_jit_dense 1 C1
cap C4 blu_jit_global 1 C4 300000000
cap C3_pass2 blu_jit_bucket 1 C3 400000000
cap C3_scatter blu_jit_scatter 33 C3 400000000
cap C3_scatter2 blu_jit_scatter 34 C3 400000000
cap C5_scatter blu_jit_scatter 1 C5 400000000
cap C5_pass2 blu_jit_global 1 C5 400000000
