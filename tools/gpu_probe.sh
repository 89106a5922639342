#!/bin/bash
# probe per-launch times of c3/c4/c2 for the default lib and variant libs given as name:lib
mkdir -p gpurun_out
out=gpurun_out/probe.txt; : > $out
for v in "def:" "$@"; do
  IFS=: read name lib <<< "$v"
  echo "== $name" >> $out
  export AIRTOPK_LIB=${lib:-paper_conf_sc_zhangnlw23_b200/libairtopk.so}
  python tools/probe_select.py --config c3 --k 1 --k 1048576 --tma 1 --tma -1 --window 1 >> $out 2>&1
  python tools/probe_select.py --config c4 --tma 1 --tma -1 >> $out 2>&1
  python tools/probe_select.py --config c2 --tma 0 >> $out 2>&1
done
