"""Print the c2 A/B results of tools/gpu_c2ab.sh (gpurun_out/c2ab)."""
import glob, json, os, re
O = "gpurun_out/c2ab"
for line in open(os.path.join(O, "batch_timing.txt")):
    if not re.search(r"Warn|rel =|med =", line):
        print(line.rstrip())
for f in sorted(glob.glob(os.path.join(O, "bench_*.json"))):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(os.path.basename(f), round(d["ms_per_step"] * 1e3, 2), "us", "frac", round(d["roofline"]["frac"], 3))
    except Exception as e:  # noqa: BLE001
        print(os.path.basename(f), "ERR", e)
