#!/bin/bash
# Round-2 first check: GPU tests, smoke, default bench (c3 + extras + per-rank proxies + cpu baseline),
# reference arm, and the multi-rank flow (2 ranks on one GPU, gloo) for the split-row and row paths.
mkdir -p gpurun_out/r02a
O=gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > $O/pytest_gpu.log
timeout 120 python __graft_entry__.py smoke > $O/smoke.log 2>&1
timeout 600 python bench.py > $O/bench_full.json 2> $O/bench_full.err
timeout 400 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
timeout 300 python bench.py --gpus 2 --dist-backend gloo --steps 20 --no-cpu --e2e-steps 1 > $O/bench_g2_c3.json 2> $O/bench_g2_c3.err
timeout 300 python bench.py --gpus 2 --dist-backend gloo --config c2 --steps 50 --no-cpu --e2e-steps 1 > $O/bench_g2_c2.json 2> $O/bench_g2_c2.err
AIRTOPK_CLUSTER_TIMING=1 timeout 120 python tools/cluster_timing.py > $O/cluster_timing.txt 2>&1
ls -la $O
