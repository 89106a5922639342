#!/bin/bash
# ncu --set full over one whole c3 select (2nd rep: sample, window, redo, trailing passes) + c4 tail
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -s 9 -c 9 -o gpurun_out/full_c3_all python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_a.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cluster_kernel -s 1 -c 1 -o gpurun_out/full_c4_tail python tools/prof_select.py --config c4 --reps 2 > gpurun_out/ncu_t.log 2>&1
