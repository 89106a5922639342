#!/bin/bash
# tests + benches + launch lists (with dram bytes) + calibration of dram byte counters on a plain copy
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
for c in c3 c2 c4 c1; do python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_$c.json 2>gpurun_out/bench_$c.err; done
for c in c3 c4 c2; do timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches_$c.csv python tools/prof_select.py --config $c --reps 3 > /dev/null 2>&1; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"copy|reduce|elementwise" -c 8 --csv --log-file gpurun_out/launches_copy.csv python -c "
import torch
x=torch.rand(1<<30, device='cuda')
y=torch.empty_like(x)
torch.cuda.synchronize()
for _ in range(2): y.copy_(x)
for _ in range(2): s=x.sum()
torch.cuda.synchronize()
" > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 8 -c 1 -o gpurun_out/full_c3_window python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_w.log 2>&1
