#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
CONFIGS="c3 c4" bash tools/gpu_libab.sh "r5::"
for c in c1 c2; do python bench.py --config $c --engine 4 --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_${c}_gs_1.json 2> gpurun_out/ab_${c}_gs_1.err; done
python tools/sample_timing.py c3 > gpurun_out/sample_timing.txt 2>&1
