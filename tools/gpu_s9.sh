mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/lp tools/ldgsts_probe.cu && timeout 40 /tmp/lp > gpurun_out/s9_ldgsts_probe.txt 2>&1
