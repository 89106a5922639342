"""Summarise gpurun_out bench JSON lines and ncu launch lists."""
import csv
import glob
import json
import os
import sys

d = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out"
for f in sorted(glob.glob(os.path.join(d, "bench_*.json"))):
    try:
        j = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(os.path.basename(f), "ERR", e)
        continue
    r = j.get("roofline") or {}
    w = j.get("whole_select", {})
    print(f"{os.path.basename(f):18s} {j['config']['workload']} value={j['value']:.4g} ms={j['ms_per_step']:.4f} "
          f"dom_frac={r.get('frac', 0):.3f} whole_frac={w.get('frac', 0):.3f} per_kernel={[round(x, 4) for x in w.get('per_kernel_ms', [])]} "
          f"clk={j.get('clocks', {}).get('sm_mhz')}")
    if "e2e" in j:
        print("   e2e", round(j["e2e"]["value"] / 1e9, 3), "Gelem/s", round(j["e2e"]["ms_per_step"], 2), "ms")
    if "cpu_baseline" in j:
        print("   cpu", j["cpu_baseline"]["value"] / 1e6, "Melem/s", j["cpu_baseline"]["sample"])
    for k, v in j.get("extras", {}).items():
        print("   extra", k, {a: (round(b, 4) if isinstance(b, float) else b) for a, b in v.items()})
for f in sorted(glob.glob(os.path.join(d, "launches_*.csv"))):
    rows = list(csv.reader(open(f)))
    try:
        hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    except IndexError:
        continue
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    print(os.path.basename(f), [(r[ki][:40].replace("void ", ""), r[vi]) for r in rows[hi + 1:hi + 9]])
