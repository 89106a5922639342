#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
CONFIGS="c3 c4 c2" bash tools/gpu_libab.sh "r7::"
python tools/sample_timing.py c3 > gpurun_out/sample_timing.txt 2>&1
python tools/pass_timing.py c4 > gpurun_out/pass_timing.txt 2>&1
