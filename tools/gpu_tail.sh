#!/bin/bash
mkdir -p gpurun_out
for c in c1 c2; do python tools/tail_timing.py $c; done > gpurun_out/tail_timing.txt 2>&1
