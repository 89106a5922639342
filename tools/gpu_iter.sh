#!/bin/bash
# iteration: batched / resident tests + fuzz, c2 stamps, c1/c2 A/B vs the previous library
O=gpurun_out/iter; rm -rf $O; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > $O/pytest.log
timeout 200 python tests/fuzz_gpu.py 150 97 > $O/fuzz.txt 2>&1
for l in paper_conf_sc_zhangnlw23_b200/libairtopk.so build_var/lib_prev.so; do
  echo "== $l" >> $O/batch_timing.txt
  AIRTOPK_LIB=$l timeout 120 python tools/batch_timing.py 100 >> $O/batch_timing.txt 2>&1
  AIRTOPK_LIB=$l timeout 120 python tools/resident_timing.py 65536 32 0 >> $O/batch_timing.txt 2>&1
done
rm -rf gpurun_out/ab2
CONFIGS="c1 c2" bash tools/gpu_libab2.sh build_var/lib_prev.so
