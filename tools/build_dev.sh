#!/bin/bash
# Developer build of libjigsaw.so with the JIG_DEV experiment knobs (env-read once
# at load: JIGSAW_STATIC_SCHEDULE, JIGSAW_UNIT_COST, JIGSAW_DBG, ...) for A/B runs:
#   JIGSAW_LIB_AB=tools/libjigsaw_dev.so python ...
# Extra defines: tools/build_dev.sh "JIG_TRACE_KB_ON=1"
set -e
cd "$(dirname "$0")/.."
D=""
for d in JIG_DEV=1 $1; do D="$D -D$d"; done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC \
  -Xcompiler -fvisibility=hidden -shared $D -o tools/libjigsaw_dev.so \
  paper_conf_icpp_zhanglyfyllq24_b200/csrc/api.cu paper_conf_icpp_zhanglyfyllq24_b200/csrc/reorder.cu \
  paper_conf_icpp_zhanglyfyllq24_b200/csrc/spmm.cu
