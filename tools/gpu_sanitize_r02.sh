#!/bin/bash
# compute-sanitizer over the round-2 engines (batched, resident, fused tail, GridSelect, p2p-free
# shard path, ablation harness): memcheck on their test files, racecheck + synccheck on subsets
O=gpurun_out/r02; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
T="tests/test_gpu_batch.py tests/test_gpu_resident.py tests/test_gpu_shard.py tests/test_gpu_ablation.py"
timeout 1800 compute-sanitizer --tool memcheck --report-api-errors no --error-exitcode 99 --print-limit 20 \
  python -m pytest $T -q -x -p no:cacheprovider > $O/sanitize_memcheck.log 2>&1
echo "memcheck ($T) exit=$?" > $O/sanitize_summary.txt
timeout 1200 compute-sanitizer --tool memcheck --report-api-errors no --error-exitcode 99 --print-limit 20 \
  python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "gridselect or window or trace or engines" > $O/sanitize_memcheck2.log 2>&1
echo "memcheck (test_gpu_parity: gridselect, window/fused tail, trace, engines) exit=$?" >> $O/sanitize_summary.txt
K="dtypes or shapes and 100 or cluster_sizes"
for tool in racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 \
    python -m pytest tests/test_gpu_batch.py tests/test_gpu_resident.py -q -x -k "dtypes" -p no:cacheprovider > $O/sanitize_$tool.log 2>&1
  echo "$tool (batched + resident dtypes) exit=$?" >> $O/sanitize_summary.txt
done
timeout 900 python tests/fuzz_gpu.py 600 2024 > $O/fuzz.txt 2>&1
echo "fuzz exit=$?" >> $O/sanitize_summary.txt
cat $O/sanitize_summary.txt; tail -3 $O/fuzz.txt
