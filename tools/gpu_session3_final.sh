# final check of this session: smoke, GPU tests, C4 bench line + ncu capture of the new front kernel
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1g_smoke.log 2>&1; tail -1 gpurun_out/r1g_smoke.log
python -m pytest tests -m gpu -q > gpurun_out/r1g_gputests.log 2>&1; tail -1 gpurun_out/r1g_gputests.log
python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/r1g_bench_C4.json 2> gpurun_out/r1g_bench_C4.err
python bench.py --steps 200 --warmup 5 > gpurun_out/r1g_bench_C2.json 2> gpurun_out/r1g_bench_C2.err
ncu --set full --clock-control none --import-source on -k regex:"blu_jit_global" -s 2 -c 1 -o gpurun_out/r1g_prof_C4 env ITERS=3 python tools/phase_probe.py C4 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r1g_launches_C2.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ls gpurun_out | grep r1g
