#!/bin/bash
mkdir -p gpurun_out
./tools/microbench_hist > gpurun_out/mb_load.txt 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_mb.csv ./tools/microbench_hist ncu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cluster_kernel -s 1 -c 1 -o gpurun_out/full_c2_tail python tools/prof_select.py --config c2 --reps 2 > gpurun_out/ncu_t.log 2>&1
