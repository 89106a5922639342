#!/bin/bash
# ncu --set full over the passes after the window pass of one c4 and one c3 select (2nd rep)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -s 11 -c 7 -o gpurun_out/full_c4_chain python tools/prof_select.py --config c4 --reps 2 > gpurun_out/ncu_a.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -s 11 -c 7 -o gpurun_out/full_c3_chain python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_b.log 2>&1
