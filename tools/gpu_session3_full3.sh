# refresh r1f: smoke, GPU tests, ncu captures + launch lists, bench lines for every config
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1f_smoke.log 2>&1; tail -2 gpurun_out/r1f_smoke.log
python -m pytest tests -m gpu -q > gpurun_out/r1f_gputests.log 2>&1; tail -2 gpurun_out/r1f_gputests.log
TAG=r1f bash tools/capture_profiles.sh all
ls gpurun_out | grep r1f | wc -l
