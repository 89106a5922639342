#!/bin/bash
# batched engine bring-up: its tests, the whole GPU suite, c2 bench + proxies, phase timing
O=gpurun_out/r02b; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_batch.py -q -x --timeout 120 2>&1 | tail -30 > $O/pytest_batch.log
timeout 900 python -m pytest tests -m gpu -q --timeout 300 2>&1 | tail -30 > $O/pytest_gpu.log
for r in 100 50 25 13; do timeout 60 python tools/batch_timing.py $r >> $O/batch_timing.txt 2>&1; done
timeout 300 python bench.py --config c2 --no-cpu --no-extras --e2e-steps 1 > $O/bench_c2.json 2> $O/bench_c2.err
timeout 120 python __graft_entry__.py smoke > $O/smoke.log 2>&1
ls -la $O
