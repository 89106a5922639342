#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
CONFIGS="c2 c1" bash tools/gpu_libab.sh "r8::"
