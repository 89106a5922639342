#!/bin/bash
# ncu launch list of the bench command itself (B200_PROFILING.md recipe: gpu__time_duration, no clock control)
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/launches_bench_c3.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu --e2e-steps 1 \
  > gpurun_out/ncu_bench.log 2>&1
