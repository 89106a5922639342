#!/bin/bash
# ncu --set full on the filter kernels (q=1) of c3 and c4
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 8 -c 1 -o gpurun_out/prof_c3_q1 python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_c3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 8 -c 1 -o gpurun_out/prof_c4_q1 python tools/prof_select.py --config c4 --reps 2 > gpurun_out/ncu_c4.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "engines or cluster or c1 or c2 or small" 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
CONFIGS="c1 c2" bash -c 'for c in $CONFIGS; do python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_$c.json 2>gpurun_out/bench_$c.err; done'
