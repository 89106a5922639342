#!/bin/bash
# iteration: GPU tests, then A/B of variant libraries on c2/c3/c4
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > $O/pytest.log
CONFIGS="c2 c3 c4" bash tools/gpu_libab2.sh build_var/lib_head.so build_var/lib_nobpdl.so
