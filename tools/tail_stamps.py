"""Per-pass timing of the fused tail kernel (CTA 0 %globaltimer: pass start, run_pass done, grid
barrier passed, scan done). AIRTOPK_TAIL_STAMPS=1 python tools/tail_stamps.py [log2 N] [K] [dist]"""
import os
import sys

os.environ["AIRTOPK_TAIL_STAMPS"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 24
k = int(sys.argv[2]) if len(sys.argv) > 2 else 1000
dist = sys.argv[3] if len(sys.argv) > 3 else "uniform"
x = torch.from_numpy(gen.keys(dist, 5, 1 << lg).reshape(1, -1)).cuda()
res = []
for rep in range(6):
    tr = torch.zeros(16 * 4 + 256, dtype=torch.int64, device="cuda")
    at.select(x, k, trace=tr)
    torch.cuda.synchronize()
    res.append(np.concatenate([tr[:64].view(16, 4).cpu().numpy(), tr[64:128].view(16, 4).cpu().numpy()], axis=1))
t = np.median(np.stack(res[2:]).astype(np.float64), axis=0)
t0 = t[t > 1e15].min()  # (rows the window pass used for other records hold small values)
print(f"N=2^{lg} K={k} {dist}: plan {at.describe(torch.float32, 1, 1 << lg, k)}")
for q in range(16):
    if t[q, 0] > 1e15:
        r = [(v - t0) / 1e3 if v > 1e15 else float("nan") for v in t[q]]
        print(f"  pass {q}: start {r[0]:7.2f}  run_pass done {r[1]:7.2f}  barrier {r[2]:7.2f}  scan {r[3]:7.2f} us"
              f"  | in run_pass: last load-iter {r[4]:7.2f} loop end {r[5]:7.2f} flush atomics {r[6]:7.2f} queues written {r[7]:7.2f}")
