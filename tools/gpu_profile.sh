#!/bin/bash
# ncu evidence for the current kernel: launch list of a short bench run and one
# --set full capture of the grouped k_spmm launch (the C2 step).  usage: TAG
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
   --log-file $OUT/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-cublas > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 \
   -o $OUT/${TAG}_grouped python tools/run_c2_batch.py > $OUT/${TAG}_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:k_spmm -s 2 -c 1 \
   -o $OUT/${TAG}_c4 python tools/run_c2_batch.py c4 > $OUT/${TAG}_ncu_c4.log 2>&1
tail -2 $OUT/${TAG}_ncu.log
ls -la $OUT | tail -5
