mkdir -p gpurun_out
T=$1
run() { v=$(env "$@" timeout 300 python bench.py --no-cpu --no-cublas --steps 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['per_launch_us'],1))"); echo "$* : $v us" >> gpurun_out/${T}_knobs.txt; }
run A=0
run JIGSAW_NO_PIECES=1
run JIGSAW_SCHED=loc
run JIGSAW_FORCE_NT=64
run JIGSAW_UNIT_COST=2
run JIGSAW_PDL=0
