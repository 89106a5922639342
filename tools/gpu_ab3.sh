#!/bin/bash
# tests + A/B of bench flags: default vs $FLAGS variants
mkdir -p gpurun_out
rm -f gpurun_out/bench_*.json
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
for c in ${CONFIGS:-c3 c4 c2}; do
  python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_${c}.json 2>gpurun_out/bench_${c}.err
  i=0
  for f in "$@"; do
    i=$((i+1))
    python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 $f > gpurun_out/bench_${c}_v$i.json 2>gpurun_out/bench_${c}_v$i.err
  done
done
