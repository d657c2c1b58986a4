# the two-stream split-pieces test against the previous device-wide 4-region workspace build (ab/libjigsaw_oldws.so) and the per-stream one
L=paper_conf_icpp_zhanglyfyllq24_b200/libjigsaw.so
cp $L /tmp/new.so; cp ab/libjigsaw_oldws.so $L; touch $L
for i in 1 2 3; do timeout 300 python -m pytest tests/test_gpu_parity.py -q -k two_streams 2>&1 | tail -1 | sed 's/^/old workspace: /'; done
cp /tmp/new.so $L; touch $L
for i in 1 2 3; do timeout 300 python -m pytest tests/test_gpu_parity.py -q -k two_streams 2>&1 | tail -1 | sed 's/^/per-stream workspace: /'; done
