cd tools/microbench
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -o smagg_bench smagg_bench.cu || exit 1
timeout 60 ./smagg_bench 1000000000 2111 4096 1024
timeout 60 ./smagg_bench 1000000000 3000 4096 1024
