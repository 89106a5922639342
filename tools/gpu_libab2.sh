#!/bin/bash
# A/B of library variants on c3/c4/c5-shard shapes: probe_select per-launch times + bench lines
# usage: tools/gpu_libab2.sh lib1 lib2 ...   (the default lib first)
O=gpurun_out/ab2; rm -rf $O; mkdir -p $O
for l in paper_conf_sc_zhangnlw23_b200/libairtopk.so "$@"; do
  n=$(basename $l .so)
  for c in ${CONFIGS:-c3 c4}; do
    AIRTOPK_LIB=$l timeout 120 python tools/probe_select.py --config $c >> $O/probe_$n.txt 2>&1
    for rep in 1 2; do
      AIRTOPK_LIB=$l timeout 300 python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > $O/bench_${n}_${c}_$rep.json 2>/dev/null
    done
  done
done
