# A/B: C2 step as 36 separate jigsaw_spmm launches in one graph (back to back) + batched
mkdir -p gpurun_out
T=$1; shift
for rep in 1 2; do for lib in "$@"; do
  JIGSAW_LIB_AB=$lib timeout 400 python bench.py --no-cpu --steps 50 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); c=d['cublas']
print('$lib rep$rep', 'batched', round(d['ms_per_step']*1e3,1), 'us  unbatched', round(c['jigsaw_unbatched_step_ms']*1e3,1), 'us  cublas batch', round(c['step_ms']*1e3,1), 'us  speedup_total_time', round(c['speedup_total_time'],3))" >> gpurun_out/${T}_unb.txt
done; done
