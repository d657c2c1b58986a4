mkdir -p gpurun_out
for cap in 0 48 200; do for wl in c2 c4; do
JIGSAW_GROUP_BPF=$cap timeout 300 python bench.py --workload $wl --steps 30 --warmup 5 --no-cpu --no-cublas > /tmp/b.json 2>/tmp/b.err
python -c "import json;b=json.load(open('/tmp/b.json'));print('bpf cap $cap MB $wl',round(b['value'],1),round(b['ms_per_step']*1e3,1),'us')" >> gpurun_out/s20_bpf.txt 2>&1 || tail -3 /tmp/b.err >> gpurun_out/s20_bpf.txt
done; done
