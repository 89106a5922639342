#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "engines or window_tail or c2_full or c1_full or cluster or distributions" 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
CONFIGS="c2 c1" bash tools/gpu_libab.sh "r9::"
CONFIGS="c3 c4" bash tools/gpu_libab.sh "bu4::" "bu8:build_var/lib_bu8.so:"
