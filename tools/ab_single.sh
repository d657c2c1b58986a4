# single-product A/B of an environment switch: graph timing of C2 points
mkdir -p gpurun_out
T=$1; shift
for env in "$@"; do echo "== $env" >> gpurun_out/${T}_single_ab.txt; env $env POINTS=0,8,9,10,15,16,26,27,33,34 REPS=3 timeout 300 python tools/single_c2.py >> gpurun_out/${T}_single_ab.txt 2>&1; done
