#!/bin/bash
# window-pass full captures (c3, c4) + A/B: direct-mode buffer passes / early ring vs HEAD
O=gpurun_out/r02final; mkdir -p $O
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 2 -c 1 -o $O/full_c3_window python tools/prof_select.py --config c3 --reps 3 > $O/ncu_c3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 2 -c 1 -o $O/full_c4_window python tools/prof_select.py --config c4 --reps 3 > $O/ncu_c4.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_ablation.py -q -x 2>&1 | tail -3 > gpurun_out/iter_pytest.log
CONFIGS="c3 c4" bash tools/gpu_libab2.sh build_var/lib_head.so build_var/lib_nodirect.so build_var/lib_noearly.so
for l in paper_conf_sc_zhangnlw23_b200/libairtopk.so build_var/lib_head.so; do
  echo "== $l" >> gpurun_out/ab2/tail_stamps.txt
  AIRTOPK_LIB=$l AIRTOPK_TAIL_STAMPS=1 timeout 120 python tools/tail_stamps.py 30 1048576 uniform >> gpurun_out/ab2/tail_stamps.txt 2>&1
  AIRTOPK_LIB=$l AIRTOPK_TAIL_STAMPS=1 timeout 120 python tools/tail_stamps.py 28 50000 adversarial >> gpurun_out/ab2/tail_stamps.txt 2>&1
done
