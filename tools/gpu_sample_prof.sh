#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sample_kernel -s 2 -c 1 -o gpurun_out/full_c2_sample python tools/prof_select.py --config c2 --reps 3 > gpurun_out/ncu_s.log 2>&1
ncu -i gpurun_out/full_c2_sample.ncu-rep --page source --csv --print-source sass > gpurun_out/src_c2_sample.csv 2>/dev/null
