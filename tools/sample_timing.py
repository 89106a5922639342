"""Phase timing of sample_kernel (debug): python tools/sample_timing.py c3"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
c = bench.CFG[cfg]
x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
tr = at.trace_buffer(c["batch"])
for _ in range(3):
    at.select(x, c["k"], trace=tr, engine=1)
torch.cuda.synchronize()
t = tr[:, 15, :7].cpu().numpy()
for r in range(min(3, len(t))):
    d = (t[r] - t[r][0]) / 1e3
    print(cfg, "row", r, "us since start: pdl_wait", d[1], "ticket", d[2], "codes", d[3], "minmax", d[5], "ranks", d[6], "done", d[4])
