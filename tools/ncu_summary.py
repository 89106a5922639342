"""Summarise ncu CSV launch lists (gpu__time_duration + dram bytes) into per-kernel rows.

    python tools/ncu_summary.py gpurun_out/launches_c3.csv [--skip N] [--count M]
"""
import csv
import sys
from collections import OrderedDict


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ix = {n: h.index(n) for n in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value")}
    launches = OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) < len(h):
            continue
        key = int(r[ix["ID"]])
        d = launches.setdefault(key, {"name": r[ix["Kernel Name"]]})
        v = float(r[ix["Metric Value"]].replace(",", ""))
        unit = r[ix["Metric Unit"]]
        if unit in ("Kbyte", "KB"):
            v *= 1e3
        elif unit in ("Mbyte", "MB"):
            v *= 1e6
        elif unit in ("Gbyte", "GB"):
            v *= 1e9
        elif unit == "usecond":
            v *= 1e3
        elif unit == "msecond":
            v *= 1e6
        d[r[ix["Metric Name"]]] = v
    return list(launches.values())


def short(name):
    n = name.replace("void ", "").replace("airtopk::", "")
    return n.split("(")[0]


if __name__ == "__main__":
    path = sys.argv[1]
    L = load(path)
    print(f"{'#':>3} {'kernel':46s} {'time_us':>9} {'dram_MB':>10} {'GB/s':>8}")
    tot_t = tot_b = 0
    for i, d in enumerate(L):
        t = d.get("gpu__time_duration.sum", 0) / 1e3
        b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        tot_t += t
        tot_b += b
        print(f"{i:3d} {short(d['name'])[:46]:46s} {t:9.1f} {b / 1e6:10.1f} {b / (t * 1e3) if t else 0:8.0f}")
    print(f"    {'total':46s} {tot_t:9.1f} {tot_b / 1e6:10.1f}")
