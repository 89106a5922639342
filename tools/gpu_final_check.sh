#!/bin/bash
# last HEAD check: the driver's round-end commands (GPU tests, smoke, default bench)
O=gpurun_out/final; rm -rf $O; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > $O/pytest_gpu.log
timeout 120 python __graft_entry__.py smoke > $O/smoke.log 2>&1
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
for c in c1 c2 c4; do timeout 300 python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > $O/bench_$c.json 2>/dev/null; done
