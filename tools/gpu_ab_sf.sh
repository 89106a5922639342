#!/bin/bash
# small-finish correctness + window-pass streaming variants
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
for sf in 0 1024; do
  for c in c3 c4; do
    AIRTOPK_SMALL_FINISH=$sf python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_${c}_sf$sf.json 2> gpurun_out/ab_${c}_sf$sf.err
  done
done
CONFIGS="c3" bash tools/gpu_libab.sh "base::" "tmaoff::--tma -1" "c16:build_var/lib_c16.so:" "c64:build_var/lib_c64.so:" "s4:build_var/lib_s4.so:"
