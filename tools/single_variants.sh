# single C2 products under forced (NT, split S) variants vs the cost model's choice
mkdir -p gpurun_out
T=$1
P="9,15,27,33"
echo "== auto" >> gpurun_out/${T}_variants.txt
POINTS=$P REPS=3 timeout 300 python tools/single_c2.py >> gpurun_out/${T}_variants.txt 2>&1
for nt in 32 64; do for s in 1 2 4 8; do
  echo "== NT=$nt S=$s" >> gpurun_out/${T}_variants.txt
  JIGSAW_FORCE_NT=$nt JIGSAW_FORCE_SPLIT=$s POINTS=$P REPS=3 timeout 300 python tools/single_c2.py >> gpurun_out/${T}_variants.txt 2>&1
done; done
