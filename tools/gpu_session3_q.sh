# N > 1 bench code path on one GPU (gloo, both ranks on cuda:0): C2 allreduce, C5 partials exchange, S1 replicas, reference arm
export BLU_BENCH_DIST_BACKEND=gloo BLU_BENCH_DEVICE=0
R="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533"
timeout 600 $R bench.py --gpus 2 --steps 3 --warmup 3 --no-e2e > gpurun_out/s3q_C2.json 2> gpurun_out/s3q_C2.err; echo "C2 rc=$?"; tail -c 600 gpurun_out/s3q_C2.json; grep -i error gpurun_out/s3q_C2.err | head -3
timeout 600 $R bench.py --gpus 2 --config C5 --rows 200000000 --steps 3 --warmup 3 --no-e2e > gpurun_out/s3q_C5.json 2> gpurun_out/s3q_C5.err; echo "C5 rc=$?"; tail -c 600 gpurun_out/s3q_C5.json; grep -i "error\|Error" gpurun_out/s3q_C5.err | head -5
timeout 600 $R bench.py --gpus 2 --config S1 --rows 10000000 --steps 3 --warmup 3 --no-e2e > gpurun_out/s3q_S1.json 2> gpurun_out/s3q_S1.err; echo "S1 rc=$?"; tail -c 300 gpurun_out/s3q_S1.json
timeout 600 $R bench.py --gpus 2 --impl reference --steps 3 --warmup 3 > gpurun_out/s3q_ref.json 2> gpurun_out/s3q_ref.err; echo "ref rc=$?"; tail -c 300 gpurun_out/s3q_ref.json
