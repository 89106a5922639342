#!/bin/bash
# iteration: GPU tests, short fuzz, c2 stamps, c2/c3/c4 bench lines + probes
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > $O/pytest.log
timeout 200 python tests/fuzz_gpu.py 150 77 > $O/fuzz.txt 2>&1
timeout 120 python tools/batch_timing.py 100 > $O/batch_timing.txt 2>&1
for c in c2 c3 c4; do timeout 120 python tools/probe_select.py --config $c >> $O/probe.txt 2>&1; done
for c in c2 c3 c4; do for rep in 1 2; do timeout 300 python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > $O/bench_${c}_$rep.json 2>/dev/null; done; done
