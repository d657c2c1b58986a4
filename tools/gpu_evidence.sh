#!/bin/bash
# One GPU session of round evidence: full bench lines (C2 default, C4), the ncu
# launch list of the default bench command, and one `ncu --set full` capture of
# the grouped k_spmm launch for C2 and for C4.   usage: tools/gpu_evidence.sh TAG
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/${TAG}_smi.txt 2>&1
timeout 600 python bench.py --detail > $OUT/${TAG}_bench_c2.json 2> $OUT/${TAG}_bench_c2.err
timeout 600 python bench.py --workload c4 --steps 30 --detail > $OUT/${TAG}_bench_c4.json 2> $OUT/${TAG}_bench_c4.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
   --log-file $OUT/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-cublas > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 \
   -o $OUT/${TAG}_c2_grouped python tools/run_c2_batch.py > $OUT/${TAG}_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 2 -c 1 \
   -o $OUT/${TAG}_c4 python tools/run_c2_batch.py c4 > $OUT/${TAG}_ncu_c4.log 2>&1
tail -2 $OUT/${TAG}_ncu.log $OUT/${TAG}_ncu_c4.log
python -c "import json;d=json.load(open('$OUT/${TAG}_bench_c2.json'));print('c2',d['value'],d['roofline'],d['cublas']['speedup_step'])"
python -c "import json;d=json.load(open('$OUT/${TAG}_bench_c4.json'));print('c4',d['value'],d['roofline'],d['cublas']['speedup_step'])"
ls -la $OUT | tail -8
