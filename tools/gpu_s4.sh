mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/gb tools/gather_bench.cu -lcuda && timeout 120 /tmp/gb > gpurun_out/s4_gather_bench.txt 2>&1
