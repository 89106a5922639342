#!/bin/bash
# quick GPU iteration: parity tests, bench (c3 + optional configs), launch list
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
python bench.py --no-extras --no-cpu --e2e-steps 1 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
for c in ${CONFIGS:-c2 c4 c1}; do python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_$c.json 2>gpurun_out/bench_$c.err; done
AIRTOPK_CLUSTER_BATCHED=1 python bench.py --config c2 --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_c2cl.json 2>gpurun_out/bench_c2cl.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c3.csv python tools/prof_select.py --config c3 --reps 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c4.csv python tools/prof_select.py --config c4 --reps 3 > /dev/null 2>&1
