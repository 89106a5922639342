"""Phase timing of the batched engine (engine 5) from per-CTA %globaltimer stamps written into the
trace buffer (csrc/engine_batch.cuh bstamp): A = sample (loads, selection), B = stream,
C = finish (slot counts, gather, window check, results, radix passes).
    python tools/batch_timing.py [rows] [n] [k] [dist]"""
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
do_flush = not (len(sys.argv) > 5 and sys.argv[5] == "noflush")
x = torch.from_numpy(gen.keys(dist, gen.config_seed("c2"), rows * n).reshape(rows, n)).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
G = torch.cuda.get_device_properties(0).multi_processor_count
acc = []
for rep in range(10):
    tr = torch.zeros(max(rows * 160 + G * 32, G * 32), dtype=torch.int64, device="cuda")
    if do_flush:
        flush.fill_(1)
    at.select(x, k, engine=5, trace=tr)
    torch.cuda.synchronize()
    t = tr[: G * 32].view(G, 32).cpu().numpy().astype(np.int64)
    t0 = t[:, 0][t[:, 0] > 0].min()
    rel = np.where(t > 0, (t - t0) / 1e3, np.nan)
    acc.append(rel)
rel = np.nanmedian(np.stack(acc[2:]), axis=0)  # [G, 16] median over reps
r = rel[: min(rows, G)]
med = lambda f: float(np.nanmedian(r[:, f]))
mx = lambda f, a=rel: float(np.nanmax(a[:, f]))
print(f"rows={rows} n={n} k={k} {dist} {'L2 flushed' if do_flush else 'no flush'}")
print(f"  A sample : loads {med(1):.2f}  select done {med(2):.2f}  end {med(3):.2f} (max {mx(3):.2f}) us")
print("  A select internals: hist " + " ".join(f"{med(16 + i):.2f}" for i in range(5)))
print(f"  barrier 1: {mx(4):.2f} | B stream end first/median/last {np.nanmin(rel[:,5]):.2f}/{np.nanmedian(rel[:,5]):.2f}/{mx(5):.2f} | C start (max) {mx(6):.2f}")
print("  C gather internals (start, counts zeroed, offsets, warp 0 entries): "
      + " ".join(f"{med(20 + i):.2f}" for i in range(4)) + f" (max {mx(23):.2f})")
print(f"  C finish : counts {med(7):.2f}  gather {med(8):.2f}  check {med(9):.2f}  results {med(10):.2f}  "
      f"pass-stamps {med(11):.2f}/{med(12):.2f}/{med(13):.2f}  end {med(14):.2f} (max {mx(14):.2f}); kernel end {mx(15):.2f} us")
slow = np.argsort(-np.nan_to_num(r[:, 14], nan=-1))[:4]
for c in slow:
    print(f"  slow CTA {c}: start C {r[c, 20]:.2f} offsets {r[c, 22]:.2f} warp0 entries {r[c, 23]:.2f} gathered {r[c, 7]:.2f} "
          f"results {r[c, 10]:.2f} end {r[c, 14]:.2f}")
