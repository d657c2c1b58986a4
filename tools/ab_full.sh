# A/B of two builds: bench C2/C4 (short) + a few single products (graph timing)
mkdir -p gpurun_out
T=$1; A=$2; B=$3
WORKLOADS='c2 c4' bash tools/ab_lib.sh $T $A $B
for l in $A $B; do echo "== $l" >> gpurun_out/${T}_single.txt; JIGSAW_LIB_AB=$l POINTS=9,15,27,33 REPS=3 timeout 300 python tools/single_c2.py >> gpurun_out/${T}_single.txt 2>&1; done
