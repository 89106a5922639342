"""Minimal driver for ncu: runs `reps` selects of one config (inputs resident, no oracle).

    ncu --set full -k regex:grid_pass_kernel ... python tools/prof_select.py --config c3 --reps 2
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="c3")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--alpha", type=int, default=0)
ap.add_argument("--window", type=int, default=0)
ap.add_argument("--tma", type=int, default=0)
ap.add_argument("--engine", type=int, default=0)
ap.add_argument("--plan-out", default=None, help="write {plan_key, launches_per_select} here (tools/make_profiles.py)")
a = ap.parse_args()
c = bench.CFG[a.config]
x = torch.from_numpy(bench.host_keys(a.config, c["n"], c["batch"])).cuda()
opts = dict(window=a.window, tma=a.tma, engine=a.engine)
if a.plan_out:
    import json
    plan = at.describe(x.dtype, c["batch"], c["n"], c["k"], **opts)
    json.dump({"plan_key": bench.plan_key(a.config, plan, opts), "launches_per_select": plan["launches"],
               "plan": plan}, open(a.plan_out, "w"))
for _ in range(a.reps):
    v, i = at.select(x, c["k"], alpha=a.alpha, **opts)
torch.cuda.synchronize()
print("done", a.config, v.shape)
