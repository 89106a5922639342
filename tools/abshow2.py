"""Summarise tools/gpu_libab2.sh output (gpurun_out/ab2)."""
import glob, json, os
O = "gpurun_out/ab2"
for f in sorted(glob.glob(os.path.join(O, "probe_*.txt"))):
    print(os.path.basename(f)); print(open(f).read().rstrip())
for f in sorted(glob.glob(os.path.join(O, "bench_*.json"))):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(os.path.basename(f), round(d["ms_per_step"] * 1e3, 2), "us  dominant frac", round(d["roofline"]["frac"], 3),
              "whole", round(d["whole_select"]["frac"], 3))
    except Exception as e:  # noqa: BLE001
        print(os.path.basename(f), "ERR", e)
