#!/bin/bash
# A/B/C: default library vs alternative builds listed in $ALTS
mkdir -p gpurun_out
rm -f gpurun_out/bench_*.json
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
for c in c3 c4 c2; do
  python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_${c}.json 2>gpurun_out/bench_${c}.err
  for a in $ALTS; do
    AIRTOPK_LIB=$PWD/paper_conf_sc_zhangnlw23_b200/libairtopk_$a.so python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_${c}_$a.json 2>gpurun_out/bench_${c}_$a.err
  done
done
python tools/tail_timing.py c4 > gpurun_out/tail_timing.txt 2>&1
