#!/bin/bash
# compute-sanitizer over the GPU parity tests: memcheck on the whole suite (CUDA API error reports off:
# the runtime's lazy module loading probes cuKernelGetFunction and reports a benign error 400),
# racecheck and synccheck on a subset of small shapes (every engine)
mkdir -p gpurun_out
rm -f gpurun_out/sanitize_*
K='small_and_ragged or window_fallback or gridselect_dtypes or (engines and normal) or concentrated'
timeout 2400 compute-sanitizer --tool memcheck --report-api-errors no --error-exitcode 99 --print-limit 20 \
  python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/sanitize_memcheck.log 2>&1
echo "memcheck (all gpu parity tests) exit=$?" >> gpurun_out/sanitize_summary.txt
for tool in racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py -q -x -k "$K" -p no:cacheprovider > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool (subset) exit=$?" >> gpurun_out/sanitize_summary.txt
done
bash tools/gpu_sample_prof.sh
