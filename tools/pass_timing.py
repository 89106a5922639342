"""Per-pass phase timing of the grid engine (debug; trace mode, which disables the small finish):
python tools/pass_timing.py c3   -> per launch q: span from the first CTA start to the scan, the
slowest CTA's streaming end, last ticket, scan, and CTA 0's streaming time (us)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
c = bench.CFG[cfg]
x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
for rep in range(3):
    tr = torch.zeros((c["batch"], 16, 10), dtype=torch.int64, device="cuda")
    at.select(x, c["k"], trace=tr, engine=1)
    torch.cuda.synchronize()
t = tr[0].cpu().numpy().astype("uint64")
base = None
for q in range(8):
    r = t[7 + q]
    if r[1] == 0:
        continue
    t0 = ~r[0] & 0xFFFFFFFFFFFFFFFF
    base = base or t0
    us = lambda v: (int(v) - int(t0)) / 1e3
    print(f"{cfg} q={q}: start {(int(t0) - int(base)) / 1e3:8.2f}  stream_end(max) {us(r[1]):7.2f}  ticket(max) {us(r[2]):7.2f}"
          f"  scan_done {us(r[3]) if r[3] else -1:7.2f}  cta0 start {us(r[4]):6.2f} stream {(int(r[5]) - int(r[4])) / 1e3:6.2f}")
