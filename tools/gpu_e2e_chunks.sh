# host-buffer pipeline: chunk count sweep (JIGSAW_HOST_CHUNKS) of the e2e leg
mkdir -p gpurun_out
for rep in 1 2; do for wl in c2 c4; do for CH in 2 4 8 16 36; do
JIGSAW_HOST_CHUNKS=$CH timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu --no-cublas > gpurun_out/ch_${wl}_$CH.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/ch_${wl}_$CH.json'));print('$wl chunks=$CH rep $rep e2e',round(d['e2e']['value'],2))"
done; done; done
