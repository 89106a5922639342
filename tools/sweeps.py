"""Paper-shaped sweeps (Figs. 6 and 7): time per select (CUDA events, mean of `reps`
selects, L2 flushed before each when the input is smaller than 256 MB) with the AUTO engine.
    python tools/sweeps.py n > profiles/r02_sweep_n.txt     # N sweep at K in {1, 32, 256, 32768, 0.1% N}
    python tools/sweeps.py k > profiles/r02_sweep_k.txt     # K sweep at N in {2^15, 2^20, 2^25, 2^30}
Columns: dist, batch, N, K, engine, us, elements/s, fraction of the 1-read roofline (measured copy
bandwidth)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
try:
    PEAK = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
except Exception:
    PEAK = 6650.0
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(x, k, reps):
    ws = torch.empty(max(1, at.workspace_bytes(x.dtype, x.shape[0], x.shape[1], k)), dtype=torch.uint8, device="cuda")
    out = (torch.empty((x.shape[0], k), dtype=x.dtype, device="cuda"),
           torch.empty((x.shape[0], k), dtype=torch.int64, device="cuda"))
    for _ in range(2):
        at.select(x, k, workspace=ws, out=out)
    torch.cuda.synchronize()
    small = x.numel() * 4 < (256 << 20)
    tot = 0.0
    for _ in range(reps):
        if small:
            flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        at.select(x, k, workspace=ws, out=out)
        e1.record()
        e1.synchronize()
        tot += e0.elapsed_time(e1)
    return tot / reps * 1e3


def row(x, dist, batch, n, k, reps):
    us = timeit(x, k, reps)
    eng = at.describe(x.dtype, batch, n, k)["engine"]
    alg = batch * n * 4 + batch * k * 12
    frac = alg / (us * 1e-6) / 1e9 / PEAK
    print(f"{dist:>11} {batch:>4} 2^{n.bit_length() - 1:<3} {k:>9} engine{eng} {us:>10.1f} us {batch * n / (us * 1e-6):>10.3e}/s"
          f"  roofline frac {frac:5.3f}", flush=True)


def keys(dist, batch, n):
    return torch.from_numpy(gen.keys(dist, 4242, batch * n).reshape(batch, n)).cuda()


mode = sys.argv[1] if len(sys.argv) > 1 else "n"
print(f"# {mode} sweep (peak {PEAK} GB/s measured copy bandwidth; roofline = one read of the keys + K x 12 B out)")
for dist in ("uniform", "normal", "adversarial"):
    if mode == "n":
        for batch in (1, 100):
            for lg in range(10, 31, 2):
                n = 1 << lg
                if batch * n > (1 << 32):
                    continue
                x = keys(dist, batch, n)
                for k in sorted({1, 32, 256, 32768, max(1, n // 1000)}):
                    if k >= n:
                        continue
                    row(x, dist, batch, n, k, 10 if batch * n < (1 << 26) else 5)
                del x
                torch.cuda.empty_cache()
    else:
        for lg in (15, 20, 25, 30):
            n = 1 << lg
            x = keys(dist, 1, n)
            for lk in range(3, 21, 2):
                k = 1 << lk
                if k >= n:
                    continue
                row(x, dist, 1, n, k, 10 if n < (1 << 26) else 5)
            del x
            torch.cuda.empty_cache()
