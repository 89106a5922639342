#!/bin/bash
# Final round-2 evidence at HEAD: the deliverable run (tools/gpu_r02_final.sh) + sanitizers/fuzz
# (tools/gpu_sanitize_r02.sh) + the binding / graph probe and the tail-mode probe.
bash tools/gpu_r02_final.sh
bash tools/gpu_sanitize_r02.sh
O=gpurun_out/r02final
timeout 300 python tools/probe_graph.py c1 c2 c3 c4 > $O/probe_graph.txt 2>&1
timeout 600 python tools/probe_tail.py > $O/probe_tail.txt 2>&1
