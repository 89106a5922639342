"""Per-launch times (CUDA events recorded by the library between its launches) of one select
configuration, for A/B probes:  python tools/probe_select.py --config c3 --k 1 --tma 1 --window 1"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="c3")
ap.add_argument("--k", type=int, action="append")
ap.add_argument("--tma", type=int, action="append")
ap.add_argument("--window", type=int, action="append")
ap.add_argument("--reps", type=int, default=5)
a = ap.parse_args()
c = bench.CFG[a.config]
x = torch.from_numpy(bench.host_keys(a.config, c["n"], c["batch"])).cuda()
for k in a.k or [c["k"]]:
    for w in a.window or [0]:
        for t in a.tma or [0]:
            opts = dict(window=w, tma=t)
            plan = at.describe(torch.float32, c["batch"], c["n"], k, **opts)
            nl = plan["launches"]
            tot = [0.0] * nl
            for r in range(a.reps + 2):
                evs = [torch.cuda.Event(enable_timing=True) for _ in range(nl + 1)]
                for e in evs:
                    e.record()
                arr = at.make_event_array(evs)
                at.select(x, k, events=arr, **opts)
                torch.cuda.synchronize()
                if r >= 2:
                    for q in range(nl):
                        tot[q] += evs[q].elapsed_time(evs[q + 1]) / a.reps
            print(f"{a.config} k={k:8d} window={w:2d} tma={t:2d} cpr={plan['ctas_per_row']:4d}  total {sum(tot)*1e3:8.1f} us  |",
                  " ".join(f"{v*1e3:.1f}" for v in tot), flush=True)
