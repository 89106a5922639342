#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over a subset of the GPU parity tests
mkdir -p gpurun_out
K='small_and_ragged or window_fallback or gridselect_dtypes or (engines and normal)'
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py -q -x -k "$K" -p no:cacheprovider > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit=$?" >> gpurun_out/sanitize_summary.txt
done
