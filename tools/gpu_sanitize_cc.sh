#!/bin/bash
# compute-sanitizer memcheck / racecheck over the CUDA-core tile paths (f3; run under gpurun).
compute-sanitizer --tool memcheck --target-processes all --print-limit 20 \
  python -m pytest -q -p no:cacheprovider tests/test_gpu_cuda_core.py > gpurun_out/r02cc_memcheck.txt 2>&1
compute-sanitizer --tool racecheck --target-processes all --print-limit 20 \
  python -m pytest -q -p no:cacheprovider tests/test_gpu_cuda_core.py -k "single_product_launch_shapes and split_k" > gpurun_out/r02cc_racecheck.txt 2>&1
