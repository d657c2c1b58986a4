#!/bin/bash
# One GPU session: bench (JSON line + per-point detail), ncu launch list, ncu full capture of k_spmm.
# usage: tools/gpu_bench.sh TAG [workload]
set -x
TAG=${1:-r01}; WL=${2:-c2}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/${TAG}_smi.txt 2>&1
timeout 600 python bench.py --workload $WL --detail > $OUT/${TAG}_bench.json 2> $OUT/${TAG}_bench.err
tail -3 $OUT/${TAG}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file $OUT/${TAG}_launches.csv python bench.py --workload $WL --steps 2 --warmup 3 --no-cpu --no-cublas > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 72 -c 36 \
   -o $OUT/${TAG}_spmm_full python bench.py --workload $WL --steps 1 --warmup 3 --no-cpu --no-cublas > $OUT/${TAG}_ncu_full.log 2>&1
tail -5 $OUT/${TAG}_ncu_full.log
ls -la $OUT
