#!/bin/bash
# Validate HEAD on one B200: gpu tests, smoke, default bench, per-config benches.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
for c in c1 c2 c3 c4; do
  python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
