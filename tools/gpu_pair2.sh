# P=256 (CTA pairs) vs P=128 with forced N tile widths on the C2 / C4 batches.
mkdir -p gpurun_out
for wl in c2 c4; do for cfg in "128 0" "256 128" "256 256"; do set -- $cfg
if [ "$2" = "0" ]; then unset JIGSAW_FORCE_NT; else export JIGSAW_FORCE_NT=$2; fi
timeout 300 python bench.py --workload $wl --panel-rows $1 --steps 50 --warmup 5 --no-cpu --no-cublas > gpurun_out/p2_${wl}_$1_$2.json 2> gpurun_out/p2_${wl}_$1_$2.err
python -c "import json;d=json.load(open('gpurun_out/p2_${wl}_$1_$2.json'));print('$wl P=$1 NT=$2',round(d['value'],1),round(d['ms_per_step']*1e3,1),'us',round(d['roofline']['frac'],3))"
done; done
unset JIGSAW_FORCE_NT
