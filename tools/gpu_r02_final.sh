#!/bin/bash
# Round-2 deliverable run: GPU tests, smoke, bench lines (default c3 + extras + proxies + cpu baseline,
# reference arm, c1/c2/c4/c5, paper path, GridSelect), the multi-rank flow on one GPU, ncu launch lists
# (with plan sidecars for profiles/traffic.json) and --set full captures of the dominant kernels.
O=gpurun_out/r02final; rm -rf $O; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 2>&1 | tail -6 > $O/pytest_gpu.log
timeout 120 python __graft_entry__.py smoke > $O/smoke.log 2>&1
timeout 900 python bench.py > $O/bench_full.json 2> $O/bench_full.err
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
for c in c1 c2 c4; do
  timeout 300 python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > $O/bench_$c.json 2> $O/bench_$c.err
done
timeout 300 python bench.py --config c3 --window -1 --no-cpu --no-extras --e2e-steps 1 > $O/bench_c3_paper.json 2> $O/bench_c3_paper.err
timeout 600 python bench.py --config c5 --no-extras --e2e-steps 1 --cpu-budget 6 > $O/bench_c5.json 2> $O/bench_c5.err
timeout 300 python bench.py --config c1 --engine 4 --no-cpu --no-extras --e2e-steps 1 > $O/bench_c1_gridselect.json 2> $O/bench_c1_gridselect.err
timeout 400 python bench.py --gpus 2 --dist-backend gloo --steps 20 --no-cpu --e2e-steps 1 > $O/bench_g2_c3.json 2> $O/bench_g2_c3.err
timeout 400 python bench.py --gpus 2 --dist-backend gloo --config c2 --steps 50 --no-cpu --e2e-steps 1 > $O/bench_g2_c2.json 2> $O/bench_g2_c2.err
# launch lists (serialised, cold cache) of the bench command itself and per config
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M --clock-control none -c 200 --csv --log-file $O/launches_bench_c3.csv \
  python bench.py --steps 2 --warmup 3 --no-extras --no-cpu --e2e-steps 1 > $O/ncu_bench.log 2>&1
for c in c1 c2 c3 c4; do
  timeout 300 ncu --metrics $M --clock-control none -c 40 --csv --log-file $O/launches_$c.csv \
    python tools/prof_select.py --config $c --reps 3 --plan-out $O/plan_$c.json > /dev/null 2>&1
done
timeout 300 ncu --metrics $M --clock-control none -c 40 --csv --log-file $O/launches_c3_paper.csv \
  python tools/prof_select.py --config c3 --reps 3 --window -1 --plan-out $O/plan_c3_paper.json > /dev/null 2>&1
timeout 300 ncu --metrics $M --clock-control none -c 60 --csv --log-file $O/launches_split_step.csv \
  python tools/split_step.py > $O/split_step.log 2>&1
# full captures of the dominant kernels
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 2 -c 1 -o $O/full_c3_window python tools/prof_select.py --config c3 --reps 3 > $O/ncu_c3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:batch_kernel -s 1 -c 1 -o $O/full_c2_batch python tools/prof_select.py --config c2 --reps 2 > $O/ncu_c2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 2 -c 1 -o $O/full_c4_window python tools/prof_select.py --config c4 --reps 3 > $O/ncu_c4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tail_kernel -s 1 -c 1 -o $O/full_c3_tail python tools/prof_select.py --config c3 --reps 2 > $O/ncu_c3t.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:resident_kernel -s 1 -c 1 -o $O/full_c1_resident python tools/prof_select.py --config c1 --reps 2 > $O/ncu_c1.log 2>&1
for r in 100 50 25 13; do python tools/batch_timing.py $r >> $O/batch_timing.txt 2>/dev/null; done
python tools/resident_timing.py 65536 32 0 >> $O/resident_timing.txt 2>/dev/null
for a in "24 1000 uniform" "28 50000 adversarial" "30 1048576 uniform"; do AIRTOPK_TAIL_STAMPS=1 python tools/tail_stamps.py $a >> $O/tail_stamps.txt 2>/dev/null; done
ls -la $O
# (compute-sanitizer runs: tools/gpu_sanitize_r02.sh; the tool was closed on this pool late in round 2)
