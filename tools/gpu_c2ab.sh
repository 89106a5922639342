#!/bin/bash
# c2 A/B: default lib vs variant libs (batched-engine tests, phase stamps, c2 bench line)
# usage: tools/gpu_c2ab.sh lib1 lib2 ...
O=gpurun_out/c2ab; rm -rf $O; mkdir -p $O
for l in paper_conf_sc_zhangnlw23_b200/libairtopk.so "$@"; do
  n=$(basename $l .so)
  echo "== $l" >> $O/batch_timing.txt
  AIRTOPK_LIB=$l timeout 300 python -m pytest tests/test_gpu_batch.py -q -x 2>&1 | tail -2 >> $O/batch_timing.txt
  AIRTOPK_LIB=$l timeout 120 python tools/batch_timing.py 100 >> $O/batch_timing.txt 2>&1
  for rep in 1 2; do
    AIRTOPK_LIB=$l timeout 300 python bench.py --config c2 --no-cpu --no-extras --e2e-steps 1 > $O/bench_${n}_$rep.json 2> $O/bench_${n}_$rep.err
  done
done
