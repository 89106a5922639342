#!/bin/bash
# Round-2 paper-shaped sweeps + ablations (long): results under gpurun_out/r02/
O=gpurun_out/r02; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python tools/sweeps.py n > $O/sweep_n.txt 2> $O/sweep_n.err
timeout 1200 python tools/sweeps.py k > $O/sweep_k.txt 2> $O/sweep_k.err
timeout 900 python tools/ablation.py > $O/ablation.txt 2> $O/ablation.err
python tools/engine_ab.py normal > $O/engine_ab_normal.txt 2>&1
python tools/engine_ab.py adversarial > $O/engine_ab_adversarial.txt 2>&1
ls -la $O
