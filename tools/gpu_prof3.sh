#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 8 -c 1 -o gpurun_out/full_c3_window_tma python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_w1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sample_kernel -s 1 -c 1 -o gpurun_out/full_c3_sample python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_s.log 2>&1
