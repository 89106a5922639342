#!/bin/bash
# A/B: default library vs an alternative build ($ALT, e.g. libairtopk_slowreg.so)
mkdir -p gpurun_out
for c in c3 c4 c2; do
  python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_${c}.json 2>gpurun_out/bench_${c}.err
  AIRTOPK_LIB=$PWD/paper_conf_sc_zhangnlw23_b200/${ALT:-libairtopk_slowreg.so} python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_${c}_alt.json 2>gpurun_out/bench_${c}_alt.err
done
timeout 600 python -m pytest tests -m gpu -q -x --timeout 300 -k "window or c3 or c4 or trace" 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
