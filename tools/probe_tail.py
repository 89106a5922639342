"""Batch-1 (and small-batch) rows with small windows: the cluster-engine tail after the window
pass vs the fused cooperative tail (AIRTOPK_NO_TAIL=1), on well-behaved rows and on rows whose
window is rejected or misses (a constant row, a mostly -inf row). Times: CUDA events around
back-to-back selects, L2 flushed in between.   python tools/probe_tail.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(x, k, reps=10):
    ts = []
    for r in range(reps + 2):
        flush.fill_(r & 1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        at.select(x, k)
        b.record()
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(a.elapsed_time(b) * 1e3)
    return float(np.median(ts))


cases = []
for lg, k in [(26, 10), (26, 1000), (28, 1000), (30, 32)]:
    cases.append((f"1 x 2^{lg} uniform K={k}", gen.uniform_f32(3, 1 << lg).reshape(1, -1), k))
cases.append(("4 x 2^26 uniform K=100", gen.uniform_f32(4, 4 << 26).reshape(4, -1), 100))
cases.append(("1 x 2^26 constant K=10", np.full((1, 1 << 26), 0.5, np.float32), 10))
m = np.full((1, 1 << 26), -np.inf, np.float32)
m[0, ::4096] = gen.uniform_f32(5, (1 << 26) // 4096)
cases.append(("1 x 2^26 mostly -inf K=10 (select max)", m, 10))
for name, xh, k in cases:
    x = torch.from_numpy(xh).cuda()
    largest = "select max" in name
    res = []
    for env in (None, "1"):
        if env:
            os.environ["AIRTOPK_NO_TAIL"] = env
        else:
            os.environ.pop("AIRTOPK_NO_TAIL", None)
        plan = at.describe(x.dtype, x.shape[0], x.shape[1], k)
        if largest:
            t = []
            for r in range(12):
                flush.fill_(r & 1)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                at.select(x, k, largest=True)
                b.record()
                torch.cuda.synchronize()
                if r >= 2:
                    t.append(a.elapsed_time(b) * 1e3)
            us = float(np.median(t))
        else:
            us = timeit(x, k)
        res.append(f"{'fused' if env else 'default'} (launches {plan['launches']}, cluster {plan['cluster_size']}) {us:8.1f} us")
    print(f"{name:42s} | " + " | ".join(res), flush=True)
os.environ.pop("AIRTOPK_NO_TAIL", None)
