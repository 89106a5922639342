#!/bin/bash
# Quick HEAD check on one B200: GPU tests, smoke, c2/c4 bench lines, batched-engine phase stamps.
O=gpurun_out/check; rm -rf $O; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -8 > $O/pytest_gpu.log
timeout 120 python __graft_entry__.py smoke > $O/smoke.log 2>&1
for c in c1 c2 c3 c4; do
  timeout 300 python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > $O/bench_$c.json 2> $O/bench_$c.err
done
for r in 100 13; do timeout 120 python tools/batch_timing.py $r >> $O/batch_timing.txt 2>&1; done
for a in "28 50000 adversarial"; do AIRTOPK_TAIL_STAMPS=1 timeout 120 python tools/tail_stamps.py $a >> $O/tail_stamps.txt 2>&1; done
