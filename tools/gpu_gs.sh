#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x --timeout 120 -k gridselect 2>&1 | tail -15 > gpurun_out/pytest_gs.log
python tools/probe_cluster.py c1 > gpurun_out/probe_gs.txt 2>&1
for c in c1 c2; do python bench.py --config $c --engine 4 --no-cpu --no-extras --e2e-steps 1 > gpurun_out/ab_${c}_gs.json 2> gpurun_out/ab_${c}_gs.err; done
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
