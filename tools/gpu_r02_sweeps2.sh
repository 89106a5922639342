#!/bin/bash
# End-of-round refresh: paper-shaped sweeps (the leaner binding and the round-2 engine changes move
# the small and mid sizes), engine A/B, a longer fuzz run — results under gpurun_out/r02s/
O=gpurun_out/r02s; rm -rf $O; mkdir -p $O
timeout 1500 python tools/sweeps.py n > $O/sweep_n.txt 2> $O/sweep_n.err
timeout 1200 python tools/sweeps.py k > $O/sweep_k.txt 2> $O/sweep_k.err
timeout 700 python tools/engine_ab.py normal > $O/engine_ab_normal.txt 2>&1
timeout 700 python tools/engine_ab.py adversarial > $O/engine_ab_adversarial.txt 2>&1
timeout 700 python tests/fuzz_gpu.py 600 777 > $O/fuzz.txt 2>&1
ls -la $O
