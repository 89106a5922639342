#!/bin/bash
# bench + launch list + ncu full of the two dominant kernels (c3)
set -x
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
for h in 0 1 2; do AIRTOPK_HMODE=$h python bench.py --no-extras --no-cpu --e2e-steps 1 > gpurun_out/bench_h$h.json 2>/dev/null; done
for c in c2 c4; do python bench.py --config $c --no-cpu --e2e-steps 1 > gpurun_out/bench_$c.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_c3.csv python tools/prof_select.py --config c3 --reps 3 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:grid_pass_kernel -s 7 -c 2 -o gpurun_out/prof_c3 python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:grid_pass_kernel -s 7 -c 4 -o gpurun_out/prof_c4 python tools/prof_select.py --config c4 --reps 2 > gpurun_out/ncu_full_c4.log 2>&1
ls -la gpurun_out
