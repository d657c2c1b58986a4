mkdir -p gpurun_out
for defs in "" "JIG_L2HINTS=1"; do
JIGSAW_NVCC_DEFINES="$defs" python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)"
for h in 0 1 2 4 3; do for wl in c4 c2; do
[ -z "$defs" ] && [ $h != 0 ] && continue
JIGSAW_L2HINTS=$h timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu --no-cublas > /tmp/b.json 2>/tmp/b.err
python -c "import json;b=json.load(open('/tmp/b.json'));print('$defs hints $h $wl',round(b['value'],1),round(b['ms_per_step']*1e3,1),'us', b['clocks'])" >> gpurun_out/s19_hints.txt 2>&1 || tail -3 /tmp/b.err >> gpurun_out/s19_hints.txt
done; done; done
python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)"
