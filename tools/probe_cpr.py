"""Select time vs CTAs per row (grid engine), for batched configs:  python tools/probe_cpr.py c2 2 4 8 16 32
(PROBE_TMA=1 forces the bulk-copy streaming path)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

cfg = sys.argv[1]
c = bench.CFG[cfg]
x = torch.from_numpy(bench.host_keys(cfg, c["n"], c["batch"])).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for cpr in [int(a) for a in sys.argv[2:]]:
    for rep in range(2):
        tot = 0.0
        for it in range(40):
            flush.fill_(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            at.select(x, c["k"], ctas_per_row=cpr, tma=int(os.environ.get("PROBE_TMA", "0")))
            e1.record()
            e1.synchronize()
            if it >= 5:
                tot += e0.elapsed_time(e1)
        print(f"{cfg} tma={os.environ.get('PROBE_TMA', '0')} cpr={cpr:4d} rep={rep} {tot / 35 * 1e3:8.1f} us", flush=True)
