# full refresh: GPU tests, ncu captures + launch lists, bench lines for every config (TAG=r1d)
python -m pytest tests -m gpu -x -q > gpurun_out/r1d_gputests.log 2>&1; tail -2 gpurun_out/r1d_gputests.log
TAG=r1d bash tools/capture_profiles.sh all
ls gpurun_out
