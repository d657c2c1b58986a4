mkdir -p gpurun_out
JIGSAW_NVCC_DEFINES="JIG_TRACE_KB_ON=1" python -c "from paper_conf_icpp_zhanglyfyllq24_b200 import _build; _build.build(force=True)"
KB=1 timeout 300 python tools/trace_single.py > gpurun_out/s8_trace_kb.txt 2>&1
