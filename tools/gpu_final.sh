# round evidence: GPU suite + smoke + default bench lines (C2, C4) + launch list +
# ncu full of the grouped k_spmm (C2, C4) + reference arm.   usage: tools/gpu_final.sh TAG
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -4 > gpurun_out/${TAG}_gpu_tests.txt
cat gpurun_out/${TAG}_gpu_tests.txt
timeout 120 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/${TAG}_smoke.txt 2>&1
tail -2 gpurun_out/${TAG}_smoke.txt
bash tools/gpu_evidence.sh $TAG
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_reference_arm.json 2> gpurun_out/${TAG}_ref.err
head -c 300 gpurun_out/${TAG}_bench_reference_arm.json
