"""Merge/scan phase timing of the cluster engine (debug): AIRTOPK_CLUSTER_TIMING=1 python tools/cluster_timing.py c1 [cs]"""
import os
import sys

os.environ["AIRTOPK_CLUSTER_TIMING"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c1"
cs = int(sys.argv[2]) if len(sys.argv) > 2 else 0
c = bench.CFG[cfg]
x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
for rep in range(3):
    tr = torch.zeros(4096 * 24, dtype=torch.int64, device="cuda")
    at.select(x, c["k"], trace=tr, engine=2, cluster_size=cs)
    torch.cuda.synchronize()
t = tr.view(-1, 24).cpu().numpy()
t = t[t[:, 1] > 0]
for r in t[:2]:
    us = lambda v: (int(v) - int(r[0])) / 1e3 if v else -1
    print(cfg, "cs", cs, "end", us(r[1]), "passes", r[3], "pass ends", [us(r[4 + i]) for i in range(4)])
    print("   pass1 B/merge/C/scan", [us(r[8 + i]) for i in range(4)], " pass2", [us(r[13 + i]) for i in range(4)])
