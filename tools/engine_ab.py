"""A/B of engines on a list of shapes (CUDA events per select, L2 flushed between selects).
    python tools/engine_ab.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

SHAPES = [(1, 1 << 12, 32), (1, 1 << 14, 32), (1, 1 << 16, 32), (1, 1 << 17, 32), (1, 1 << 18, 64), (1, 1 << 19, 256),
          (1, 1 << 20, 256), (1, 1 << 22, 1000), (1, 1 << 24, 1000),
          (100, 1 << 12, 32), (100, 1 << 14, 32), (100, 1 << 16, 256), (1000, 1 << 12, 32),
          (100, 1 << 18, 256), (100, 1 << 20, 32768),
          (4, 1 << 20, 100), (16, 1 << 18, 64), (13, 1 << 20, 256), (100, 1 << 20, 256), (100, 1 << 20, 32),
          (1000, 1 << 16, 32)]
VARIANTS = {"auto": {}, "batch": {"engine": 5}, "resident": {"engine": 6}, "cluster": {"engine": 2},
            "grid paper": {"window": -1, "engine": 1}, "grid+window": {"window": 1, "engine": 1}}
if os.environ.get("AB_ALL"):
    VARIANTS.update({"grid+window(tail)": {"window": 1}})
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(x, k, kw, reps=30):
    try:
        for _ in range(3):
            at.select(x, k, **kw)
        torch.cuda.synchronize()
    except Exception as e:  # noqa: BLE001
        return None
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


DIST = sys.argv[1] if len(sys.argv) > 1 else "normal"
for batch, n, k in (SHAPES if len(sys.argv) < 3 else [s for s in SHAPES if s[0] >= int(sys.argv[2])]):
    x = torch.from_numpy(gen.keys(DIST, 5, batch * n).reshape(batch, n)).cuda()
    d = at.describe(torch.float32, batch, n, k)
    res = {name: timeit(x, k, kw) for name, kw in VARIANTS.items()}
    print(f"{DIST[:4]} {batch:5d} x 2^{n.bit_length() - 1:2d} k={k:5d} auto=engine{d['engine']}: " +
          "  ".join(f"{name} {v:7.1f}" if v is not None else f"{name}    n/a" for name, v in res.items()), flush=True)
