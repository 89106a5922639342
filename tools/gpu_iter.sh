#!/bin/bash
# one iteration: GPU tests of the touched engines, tail probe, fused-tail CTA-count sweep on c4
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "tail" 2>&1 | tail -5 > $O/pytest.log
timeout 600 python tools/probe_tail.py > $O/probe_tail.txt 2>&1
for g in 296 148 64 32 16; do
  echo "== AIRTOPK_TAIL_CTAS=$g" >> $O/tail_ctas.txt
  AIRTOPK_TAIL_CTAS=$g timeout 120 python tools/tail_stamps.py 28 50000 adversarial >> $O/tail_ctas.txt 2>&1
  AIRTOPK_TAIL_CTAS=$g timeout 120 python tools/probe_select.py --config c4 >> $O/tail_ctas.txt 2>&1
done
