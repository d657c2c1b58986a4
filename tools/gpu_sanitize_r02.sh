#!/bin/bash
# compute-sanitizer memcheck over the round-2 GPU paths (run under gpurun).
compute-sanitizer --tool memcheck --target-processes all --print-limit 20 \
  python -m pytest -q -p no:cacheprovider tests/test_gpu_bench_configs.py \
  -k "c_dtype or concurrent or many_replays or dynamic_scheduler" > gpurun_out/r02_memcheck_a.txt 2>&1
compute-sanitizer --tool memcheck --target-processes all --print-limit 20 \
  python -m pytest -q -p no:cacheprovider tests/test_gpu_parity.py \
  -k "row_clustered or grouped_split_pieces or spmm_kernel_variants or pair_panels_bit_exact" > gpurun_out/r02_memcheck_b.txt 2>&1
compute-sanitizer --tool racecheck --target-processes all --print-limit 20 \
  python -m pytest -q -p no:cacheprovider tests/test_gpu_parity.py -k "integer_inputs_bit_exact" > gpurun_out/r02_racecheck.txt 2>&1
