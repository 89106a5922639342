"""Select time vs engine / cluster size for a small-row config:  python tools/probe_cluster.py c1"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c1"
c = bench.CFG[cfg]
x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for eng, cs in [(2, 4), (2, 8), (2, 16), (1, 0), (4, 0)]:
    tot = 0.0
    for it in range(60):
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        at.select(x, c["k"], engine=eng, cluster_size=cs)
        e1.record()
        e1.synchronize()
        if it >= 10:
            tot += e0.elapsed_time(e1)
    print(f"{cfg} engine={eng} cs={cs:2d} {tot / 50 * 1e3:8.1f} us", flush=True)
