"""Per-CTA timing of the cluster engine (debug aid): python tools/tail_timing.py c2"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
c = bench.CFG[cfg]
x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
tr = torch.zeros(4096 * 8, dtype=torch.int64, device="cuda")
for w in (0, 1):
    for _ in range(3):
        at.select(x, c["k"], trace=tr, window=w if w else 0)
    torch.cuda.synchronize()
    t = tr.view(-1, 8).cpu().numpy()
    t = t[t[:, 1] > 0]
    d = (t[:, 1] - t[:, 0]) / 1e3
    print(cfg, "window" if w else "auto", at.describe(torch.float32, c["batch"], c["n"], c["k"]),
          "CTAs", len(t), "dur_us min/med/max", d.min(), np.median(d), d.max(), "rows", t[:, 2].sum(),
          "passes max", t[:, 3].max(), "span_us", (t[:, 1].max() - t[:, 0].min()) / 1e3)
    r0 = t[0]
    print("   cta0 pass ends (us from start):", [(r0[4 + i] - r0[0]) / 1e3 for i in range(4) if r0[4 + i] > 0])
    tr.zero_()
