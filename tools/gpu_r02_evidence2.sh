#!/bin/bash
# Final round-2 evidence at HEAD (compute-sanitizer is closed on the pool): the deliverable run
# (tools/gpu_r02_final.sh: tests, smoke, every bench line, reference arm, multi-rank flow, ncu launch
# lists + full captures, phase timings), a fuzz run and the two probes.
bash tools/gpu_r02_final.sh
O=gpurun_out/r02final
timeout 400 python tests/fuzz_gpu.py 300 4242 > $O/fuzz.txt 2>&1
timeout 300 python tools/probe_graph.py c1 c2 c3 c4 > $O/probe_graph.txt 2>&1
timeout 600 python tools/probe_tail.py > $O/probe_tail.txt 2>&1
