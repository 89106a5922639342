#!/bin/bash
# A/B: histogram copies of the bulk-copy filter passes (paper path: --window -1), c3 / c4 / c3-adversarial-like
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
for l in paper_conf_sc_zhangnlw23_b200/libairtopk.so build_var/lib_hc2.so; do
  echo "== $l" >> $O/probe.txt
  for c in c3 c4; do AIRTOPK_LIB=$l timeout 200 python tools/probe_select.py --config $c --window -1 >> $O/probe.txt 2>&1; done
  AIRTOPK_LIB=$l timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tma or paper or trace" 2>&1 | tail -1 >> $O/probe.txt
done
