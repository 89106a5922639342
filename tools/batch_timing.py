"""Phase timing of the batched engine (engine 5): per-CTA %globaltimer stamps written into the trace
buffer — [0] start, [1] sampling done, [2] after grid barrier 1, [3] streaming done, [4] after
barrier 2, [5] finish done.  python tools/batch_timing.py [rows] [n] [k] [dist]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

rows = int(sys.argv[1]) if len(sys.argv) > 1 else 100
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 20
k = int(sys.argv[3]) if len(sys.argv) > 3 else 256
dist = sys.argv[4] if len(sys.argv) > 4 else "normal"
x = torch.from_numpy(gen.keys(dist, gen.config_seed("c2"), rows * n).reshape(rows, n)).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
res = []
for rep in range(8):
    tr = torch.zeros(max(rows * 160, 148 * 8), dtype=torch.int64, device="cuda")
    flush.fill_(1)
    at.select(x, k, engine=5, trace=tr)
    torch.cuda.synchronize()
    t = tr[: 148 * 8].view(148, 8).cpu().numpy()[:, :6].astype(np.int64)
    t0 = t[:, 0].min()
    res.append([(t[:, f].max() - t0) / 1e3 for f in range(6)] + [(t[:, 0].max() - t0) / 1e3, (t[:, 3].min() - t0) / 1e3])
r = np.median(np.array(res[2:]), axis=0)
print(f"rows={rows} n={n} k={k} {dist}: last CTA start {r[6]:.2f} us | sampled {r[1]:.2f} | barrier1 {r[2]:.2f} | "
      f"streamed first/last {r[7]:.2f}/{r[3]:.2f} | barrier2 {r[4]:.2f} | finished {r[5]:.2f} us")
