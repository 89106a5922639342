#!/bin/bash
# A/B: samples per row of the batched engine (len/128 = 8K for c2 vs len/256 = 4K)
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
for d in 128 64; do
  echo "== AIRTOPK_BATCH_SAMP_DIV=$d" >> $O/ab.txt
  AIRTOPK_BATCH_SAMP_DIV=$d timeout 120 python tools/batch_timing.py 100 2>&1 | grep -v "Warn\|rel =\|med =\|slow CTA" >> $O/ab.txt
  for rep in 1 2; do AIRTOPK_BATCH_SAMP_DIV=$d timeout 300 python bench.py --config c2 --no-cpu --no-extras --e2e-steps 1 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('c2', d['ms_per_step']*1e3, d['roofline']['frac'])" >> $O/ab.txt; done
  AIRTOPK_BATCH_SAMP_DIV=$d timeout 600 python -m pytest tests/test_gpu_batch.py -q -x 2>&1 | tail -1 >> $O/ab.txt
done
