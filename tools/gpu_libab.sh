#!/bin/bash
# A/B of compile-time variants: tools/gpu_libab.sh "name:lib:benchflags" ...  (CONFIGS env: configs)
mkdir -p gpurun_out
for c in ${CONFIGS:-c3 c4 c2}; do
  for v in "$@"; do
    IFS=: read name lib flags <<< "$v"
    for rep in 1 2; do
      AIRTOPK_LIB=${lib:-paper_conf_sc_zhangnlw23_b200/libairtopk.so} python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 $flags > gpurun_out/ab_${c}_${name}_$rep.json 2>gpurun_out/ab_${c}_${name}_$rep.err
    done
  done
done
