mkdir -p gpurun_out
export POINTS=3,9,15,21,27,33 REPS=3
timeout 300 python tools/single_c2.py > gpurun_out/s21_single_default.txt 2>&1
JIGSAW_NO_BPF=1 timeout 300 python tools/single_c2.py > gpurun_out/s21_single_nobpf.txt 2>&1
JIGSAW_NO_CTAB=1 timeout 300 python tools/single_c2.py > gpurun_out/s21_single_noctab.txt 2>&1
