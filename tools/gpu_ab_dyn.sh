#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
python tools/pass_timing.py c3 > gpurun_out/pass_timing.txt 2>&1
CONFIGS="c3 c4" bash tools/gpu_libab.sh "dyn::" "h1m:build_var/lib_h1m.so:" "h2k:build_var/lib_h2k.so:"
