#!/bin/bash
# c2 iteration: batched-engine tests, phase stamps, bench line.
O=gpurun_out/c2; rm -rf $O; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_batch.py -q -x --timeout 300 2>&1 | tail -4 > $O/pytest_batch.log
for r in 100 13; do timeout 120 python tools/batch_timing.py $r >> $O/batch_timing.txt 2>&1; done
timeout 300 python bench.py --config c2 --no-cpu --no-extras --e2e-steps 1 > $O/bench_c2.json 2> $O/bench_c2.err
