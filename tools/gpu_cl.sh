#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
for cs in 16 4; do python tools/cluster_timing.py c1 $cs; done > gpurun_out/cluster_timing.txt 2>&1
python tools/probe_cluster.py c1 >> gpurun_out/cluster_timing.txt 2>&1
for c in c1 c2; do python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_${c}_cl.json 2> gpurun_out/ab_${c}_cl.err; done
