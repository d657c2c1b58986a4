# A/B of compile-time variants: bench C2 / C4 + single-product events per variant
# usage: tools/gpu_ab.sh TAG "DEFINES1" "DEFINES2" ...
mkdir -p gpurun_out
TAG=$1; shift
i=0
for defs in "$@"; do
  JIGSAW_NVCC_DEFINES="$defs" python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)" || { echo "build failed: $defs"; continue; }
  echo "== variant $i: $defs" >> gpurun_out/${TAG}_ab.txt
  timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu --no-cublas > /tmp/c2.json 2>/dev/null
  timeout 300 python bench.py --workload c4 --steps 20 --warmup 5 --no-cpu --no-cublas > /tmp/c4.json 2>/dev/null
  python -c "import json;a=json.load(open('/tmp/c2.json'));b=json.load(open('/tmp/c4.json'));print('C2',round(a['value'],1),round(a['ms_per_step']*1e3,2),'us  C4',round(b['value'],1),round(b['ms_per_step']*1e3,1),'us')" >> gpurun_out/${TAG}_ab.txt 2>&1
  POINTS=0,9,15,21,27,33 REPS=5 timeout 300 python tools/single_c2.py >> gpurun_out/${TAG}_ab.txt 2>&1
  i=$((i+1))
done
python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)"
