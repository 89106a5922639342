"""Phase timing of the resident-cluster engine (engine 6): per-CTA %globaltimer stamps in the trace
buffer. python tools/resident_timing.py [n] [k] [cs] [dist] [noflush]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 16
k = int(sys.argv[2]) if len(sys.argv) > 2 else 32
cs = int(sys.argv[3]) if len(sys.argv) > 3 else 0
dist = sys.argv[4] if len(sys.argv) > 4 else "uniform"
do_flush = not (len(sys.argv) > 5 and sys.argv[5] == "noflush")
x = torch.from_numpy(gen.keys(dist, gen.config_seed("c1"), n).reshape(1, n)).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
acc, ev = [], []
for rep in range(20):
    tr = torch.zeros(4096, dtype=torch.int64, device="cuda")
    if do_flush:
        flush.fill_(1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    at.select(x, k, engine=6, cluster_size=cs, trace=tr)
    e1.record()
    torch.cuda.synchronize()
    ev.append(e0.elapsed_time(e1) * 1e3)
    t = tr[:16 * 16].view(16, 16).cpu().numpy().astype(np.int64)
    t0 = t[:, 0][t[:, 0] > 0].min()
    acc.append(np.where(t > 0, (t - t0) / 1e3, np.nan))
rel = np.nanmedian(np.stack(acc[5:]), axis=0)
names = ["start", "loaded", "h0", "sync0", "scan0", "h1", "sync1", "scan1", "h2", "sync2", "scan2", "finpass",
         "finsync", "select", "end"]
print(f"n={n} k={k} cs={cs} {dist} {'flushed' if do_flush else 'noflush'}: event {np.median(ev[5:]):.2f} us")
print("  CTA0: " + "  ".join(f"{nm} {rel[0, i]:.2f}" for i, nm in enumerate(names) if not np.isnan(rel[0, i])))
print("  max : " + "  ".join(f"{nm} {np.nanmax(rel[:, i]):.2f}" for i, nm in enumerate(names)
                             if not np.all(np.isnan(rel[:, i]))))
