"""Top stall instructions of an ncu source page (SASS): python tools/ncu_src_top.py src.csv [N]"""
import csv
import sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
h = rows[1]
data = rows[2:]
isrc, iss, iex = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
reasons = [x for x in h if x.startswith("stall_") and "Not Issued" not in x]
tot = sum(int(r[iss]) for r in data)
print("samples", tot, "inst", sum(int(r[iex]) for r in data))
for k, r in enumerate(data):
    r.append(k)
for r in sorted(data, key=lambda r: -int(r[iss]))[:n]:
    br = sorted(((int(r[h.index(x)]), x[6:]) for x in reasons), reverse=True)[:3]
    print(f"{r[-1]:5d} {int(r[iss]):6d} {int(r[iex]):9d} {r[isrc][:60]:60s}", " ".join(f"{b}:{v}" for v, b in br if v))
