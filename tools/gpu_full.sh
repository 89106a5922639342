#!/bin/bash
# Round deliverable run: gpu tests, smoke, full bench (default c3 + extras + cpu baseline), reference
# arm, per-config bench lines (c1..c5, GridSelect on c1/c2), ncu launch lists and --set full captures.
mkdir -p gpurun_out
rm -f gpurun_out/bench_*.json gpurun_out/*.ncu-rep gpurun_out/launches_*.csv gpurun_out/ab_*
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt
timeout 900 python -m pytest tests -m gpu -q --timeout 300 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in c1 c2 c3 c4; do
  python bench.py --config $c --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
for c in c1 c2; do
  python bench.py --config $c --engine 4 --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_${c}_gridselect.json 2> gpurun_out/bench_${c}_gridselect.err
done
python bench.py --config c3 --window -1 --no-cpu --no-extras --e2e-steps 1 > gpurun_out/bench_c3_paper.json 2> gpurun_out/bench_c3_paper.err
timeout 600 python bench.py --config c5 --no-extras --e2e-steps 1 --cpu-budget 5 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
python tools/ablation.py > gpurun_out/ablation.txt 2>&1
# launch lists (serialised, cold-cache): window path and paper path
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c3.csv python tools/prof_select.py --config c3 --reps 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c3_paper.csv python tools/prof_select.py --config c3 --reps 3 --window -1 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c4.csv python tools/prof_select.py --config c4 --reps 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_c2.csv python tools/prof_select.py --config c2 --reps 3 > /dev/null 2>&1
# one full capture of the dominant kernel per path (window pass; paper pass 1 and 2; c4 window pass)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 8 -c 1 -o gpurun_out/full_c3_window python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_w.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 7 -c 2 -o gpurun_out/full_c3_paper python tools/prof_select.py --config c3 --reps 2 --window -1 > gpurun_out/ncu_p.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_kernel -s 10 -c 1 -o gpurun_out/full_c3_q1 python tools/prof_select.py --config c3 --reps 2 > gpurun_out/ncu_q1.log 2>&1
ncu -i gpurun_out/full_c3_window.ncu-rep --page source --csv --print-source sass > gpurun_out/src_c3_window.csv 2>/dev/null
ls -la gpurun_out | tail -40
