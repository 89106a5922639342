#!/bin/bash
# sample timing + f16/bf16 benches (adversarial regression check)
mkdir -p gpurun_out
rm -f gpurun_out/bench_*.json
for c in c3 c4 c2; do python tools/sample_timing.py $c; done > gpurun_out/sample_timing.txt 2>&1
for c in ${CONFIGS:-c4 c3}; do
  i=0
  for f in "$@"; do
    i=$((i+1))
    python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 $f > gpurun_out/bench_${c}_v$i.json 2>gpurun_out/bench_${c}_v$i.err
  done
done
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
