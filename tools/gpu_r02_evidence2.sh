#!/bin/bash
# Final round-2 evidence at HEAD (compute-sanitizer is closed on the pool): the deliverable run
# (tools/gpu_r02_final.sh: tests, smoke, every bench line, reference arm, multi-rank flow, ncu launch
# lists + full captures, phase timings), a fuzz run and the two probes. The ncu reports are
# summarised ON the box (tools/make_profiles.py) and removed: gpurun returns <= 64 MiB.
bash tools/gpu_r02_final.sh
O=gpurun_out/r02final
timeout 400 python tests/fuzz_gpu.py 300 4242 > $O/fuzz.txt 2>&1
timeout 300 python tools/probe_graph.py c1 c2 c3 c4 > $O/probe_graph.txt 2>&1
timeout 600 python tools/probe_tail.py > $O/probe_tail.txt 2>&1
timeout 300 ncu -i $O/full_c3_window.ncu-rep --page source --csv --print-source sass > $O/src_c3_window.csv 2>/dev/null
python tools/ncu_src_top.py $O/src_c3_window.csv 30 > $O/src_top_c3_window.txt 2>&1
rm -f $O/src_c3_window.csv
python tools/make_profiles.py r02 $O > $O/make_profiles.log 2>&1
mkdir -p gpurun_out/profiles_box && cp profiles/r02_* profiles/traffic.json gpurun_out/profiles_box/
rm -f $O/*.ncu-rep
du -sh gpurun_out
