#!/bin/bash
# A/B of the buffer-pass active-CTA knob (AIRTOPK_BUF_PER_CTA) + gpu tests + sample phase timing
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
for c in c3 c4 c2; do
  for b in 0 1024 4096 16384; do
    AIRTOPK_BUF_PER_CTA=$b python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_${c}_$b.json 2> gpurun_out/ab_${c}_$b.err
  done
done
for c in c3 c4 c2; do python tools/sample_timing.py $c; done > gpurun_out/sample_timing.txt 2>&1
