python -m pytest tests -m gpu -q > gpurun_out/r02fz_gpu_tests.txt 2>&1; tail -3 gpurun_out/r02fz_gpu_tests.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02fz_smoke.txt 2>&1; tail -2 gpurun_out/r02fz_smoke.txt
bash tools/gpu_evidence_r02.sh r02fz
