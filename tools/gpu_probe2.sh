#!/bin/bash
mkdir -p gpurun_out
for c in c3 c4; do python tools/pass_timing.py $c; done > gpurun_out/pass_timing.txt 2>&1
python bench.py --config c2 --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_c2_cpr8.json 2> gpurun_out/ab_c2_cpr8.err
timeout 600 python bench.py --config c5 --no-extras --e2e-steps 1 --cpu-budget 5 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
