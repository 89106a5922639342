#!/bin/bash
# one iteration: GPU parity tests, c3/c4 per-launch probes and bench lines
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q -x 2>&1 | tail -5 > $O/pytest.log
for c in c3 c4; do timeout 120 python tools/probe_select.py --config $c >> $O/probe.txt 2>&1; done
for c in c3 c4; do for rep in 1 2; do timeout 300 python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > $O/bench_${c}_$rep.json 2>/dev/null; done; done
