#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab_*
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
for c in c3 c4 c2; do
  python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_${c}_new.json 2> gpurun_out/ab_${c}_new.err
done
python tools/probe_cpr.py c2 2 4 8 16 32 64 > gpurun_out/probe_cpr.txt 2>&1
