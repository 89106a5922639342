#!/bin/bash
# ncu --set full captures of the dominant kernels of c4 and c2, and the c4 launch list
mkdir -p gpurun_out
rm -f gpurun_out/*.ncu-rep gpurun_out/launches_*.csv
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 8 -c 1 -o gpurun_out/full_c4_window python tools/prof_select.py --config c4 --reps 2 > gpurun_out/ncu_c4w.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 1 -c 1 -o gpurun_out/full_c2_window python tools/prof_select.py --config c2 --reps 2 > gpurun_out/ncu_c2w.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c4.csv python tools/prof_select.py --config c4 --reps 3 > /dev/null 2>&1
