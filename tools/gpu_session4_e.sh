# session 4: HOT_REG=1 by default — smoke, GPU tests, bench lines, C4 ncu capture
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1i_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r1i_smoke.log
python -m pytest tests -m gpu -q > gpurun_out/r1i_gputests.log 2>&1; tail -1 gpurun_out/r1i_gputests.log
python bench.py --config C4 --steps 10 --warmup 3 > gpurun_out/r1i_bench_C4.json 2> gpurun_out/r1i_bench_C4.err
python bench.py --steps 200 --warmup 5 > gpurun_out/r1i_bench_C2.json 2> gpurun_out/r1i_bench_C2.err
ncu --set full --clock-control none --import-source on -k regex:"blu_jit_global" -s 2 -c 1 -o gpurun_out/r1i_prof_C4 env ITERS=3 python tools/phase_probe.py C4 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r1i_launches_C4.csv python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ls gpurun_out | grep r1i
