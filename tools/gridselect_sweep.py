"""GridSelect (shared queue, engine 4) vs its per-thread-queue variant (engine 7, the Fig. 11
ablation) vs the radix path (AUTO) over K, on the paper's N values (Fig. 6) —
the "GridSelect is faster when K < 256" comparison. CUDA events per select, L2 flushed.
    python tools/gridselect_sweep.py [dist ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(x, k, kw, reps=20):
    for _ in range(3):
        at.select(x, k, **kw)
    torch.cuda.synchronize()
    tot = 0.0
    for _ in range(reps):
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        at.select(x, k, **kw)
        e1.record()
        e1.synchronize()
        tot += e0.elapsed_time(e1)
    return tot / reps * 1e3


dists = sys.argv[1:] or ["uniform", "normal", "adversarial"]
print("# time per select in us (L2 flushed before each): GridSelect shared queue | per-thread queues | AIR Top-K (auto)")
for dist in dists:
    for batch, n in ((1, 1 << 15), (1, 1 << 20), (1, 1 << 25), (100, 1 << 15), (100, 1 << 20)):
        x = torch.from_numpy(gen.keys(dist, 9, batch * n).reshape(batch, n)).cuda()
        for k in (8, 32, 128, 256, 512, 1024, 2048):
            g = timeit(x, k, {"engine": 4})
            t = timeit(x, k, {"engine": 7})
            r = timeit(x, k, {})
            print(f"{dist:11s} batch {batch:3d} N 2^{n.bit_length() - 1:2d} K {k:5d}: shared {g:8.1f}  per-thread {t:8.1f}"
                  f"  (shared/per-thread {t / g:4.2f}x)  radix {r:8.1f}  -> {'GridSelect' if g < r else 'radix'}",
                  flush=True)
        del x
