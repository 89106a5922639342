#!/bin/bash
# iteration: GPU tests + fuzz, fused-tail stamps, c3/c4 A/B vs a variant library
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > $O/pytest.log
timeout 200 python tests/fuzz_gpu.py 150 91 > $O/fuzz.txt 2>&1
for a in "28 50000 adversarial" "30 1048576 uniform"; do AIRTOPK_TAIL_STAMPS=1 timeout 120 python tools/tail_stamps.py $a >> $O/tail_stamps.txt 2>&1; done
CONFIGS="c3 c4" bash tools/gpu_libab2.sh build_var/lib_noident.so
