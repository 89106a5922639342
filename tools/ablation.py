"""Paper ablations on one B200 (SURVEY §2.4 E6 / Fig. 9, and the Table 3 shape):

  python tools/ablation.py > profiles/r01_ablation.txt

* Fig. 9: the adaptive strategy on radix-adversarial rows (the first M bits shared,
  P:231): the paper's passes only (window off) with alpha = 128 (adaptive), alpha = 1 (always
  buffer, "without adaptive") and alpha >= N (never buffer). CUDA events, mean of 20 selects.
* Table 3 shape: N = 2^30 uniform, K = 2048, paper's passes: per-launch times
  (events between launches) and their shares, next to the window path.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402


def timed(x, k, reps=20, **kw):
    for _ in range(3):
        at.select(x, k, **kw)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        at.select(x, k, **kw)
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3  # us


def per_launch(x, k, reps=10, **kw):
    plan = at.describe(x.dtype, x.shape[0], x.shape[1], k, **kw)
    nl = plan["launches"]
    tot = [0.0] * nl
    for r in range(reps + 2):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(nl + 1)]
        for e in evs:
            e.record()
        at.select(x, k, events=at.make_event_array(evs), **kw)
        torch.cuda.synchronize()
        if r >= 2:
            for q in range(nl):
                tot[q] += evs[q].elapsed_time(evs[q + 1]) * 1e3 / reps
    return tot


print("# Fig. 9 ablation (paper's passes, window off): time per select in us")
print(f"{'M':>3} {'N':>6} {'K':>6} {'adaptive a=128':>15} {'always a=1':>11} {'never a>=N':>11} {'always/adaptive':>16}")
for m in (10, 20):
    for lg in (20, 24, 28):
        n = 1 << lg
        x = torch.from_numpy(gen.adversarial_f32(900 + m, n, m_bits=m).reshape(1, n)).cuda()
        k = 2048
        ta = timed(x, k, window=-1, alpha=128)
        t1 = timed(x, k, window=-1, alpha=1)
        tn = timed(x, k, window=-1, alpha=1 << 40)
        print(f"{m:>3} 2^{lg:<4} {k:>6} {ta:>15.1f} {t1:>11.1f} {tn:>11.1f} {t1 / ta:>16.2f}", flush=True)
        del x
        torch.cuda.empty_cache()

print()
print("# Fig. 10 ablation (P:305-309): early stopping on vs off, uniform rows, paper's passes (window off), us")
print(f"{'N':>6} {'K':>7} {'early stop on':>14} {'off':>9} {'off/on':>7}")
for lg, k in ((20, 32), (24, 256), (28, 2048), (30, 2048)):
    n = 1 << lg
    x = torch.from_numpy(gen.uniform_f32(gen.config_seed("c3"), n).reshape(1, n)).cuda()
    ton = timed(x, k, window=-1)
    toff = timed(x, k, window=-1, early_stop=-1)
    print(f"2^{lg:<4} {k:>7} {ton:>14.1f} {toff:>9.1f} {toff / ton:>7.3f}", flush=True)
    del x
    torch.cuda.empty_cache()

print()
print("# Table 3 shape: N = 2^30 uniform, K = 2048 (paper: kernel 1 49.29 %, 2 50.30 %, 3 0.29 %, last 0.12 %)")
n = 1 << 30
x = torch.from_numpy(gen.uniform_f32(gen.config_seed("c3"), n).reshape(1, n)).cuda()
for w, name in ((-1, "paper's passes (window off)"), (0, "default (window)")):
    t = per_launch(x, 2048, window=w)
    s = sum(t)
    print(f"{name}: total {s:.1f} us |", " ".join(f"{v:.1f} ({100 * v / s:.2f}%)" for v in t))

print()
print("# Kernel organisation (P:146-156, airtopk_select_ablation: plain kernels, scalar loads): us per select")
print("# design 0 naive (Fig. 2: 4 kernels per iteration), 1 iteration-fused (Fig. 3), 2 fused last filter (P:156)")


def timed_abl(x, k, design, b, reps=10):
    for _ in range(2):
        at.select_ablation(x, k, design, b)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        _, _, nk = at.select_ablation(x, k, design, b)
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3, nk


print(f"{'data':>12} {'N':>6} {'K':>6} " + " ".join(f"{nm:>22}" for nm in
      ("naive b=8", "naive b=11", "fused b=8", "fused b=11", "fused+lastfilter b=11")))
for dist, m in (("uniform", 20), ("adversarial", 20)):
    for lg in (20, 26, 28):
        n = 1 << lg
        x = torch.from_numpy(gen.keys(dist, 905, n, m_bits=m).reshape(1, n)).cuda()
        k = 2048
        cells = []
        for design, b in ((0, 8), (0, 11), (1, 8), (1, 11), (2, 11)):
            t, nk = timed_abl(x, k, design, b)
            cells.append(f"{t:>12.1f} ({nk:2d} kern)")
        print(f"{dist:>12} 2^{lg:<4} {k:>6} " + " ".join(f"{c:>22}" for c in cells), flush=True)
        del x
        torch.cuda.empty_cache()

print()
print("# Sorted output option (one extra launch): us per select, batch 100 x 2^20 normal")
x = torch.from_numpy(gen.normal_f32(906, 100 << 20).reshape(100, 1 << 20)).cuda()
for k in (32, 256, 4096):
    print(f"K {k:5d}: unordered {timed(x, k):8.1f}  sorted {timed(x, k, sorted=True):8.1f}", flush=True)
