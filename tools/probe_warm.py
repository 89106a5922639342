import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, gen, paper_conf_sc_zhangnlw23_b200 as at
n, k = 1 << 16, 32
x1 = gen.config_keys("c1").reshape(1, n)
for batch in (1, 2, 4, 8):
    x = torch.from_numpy(np.repeat(x1, batch, axis=0)).cuda()
    tr = torch.zeros(batch * 160 + 4096, dtype=torch.int64, device="cuda")
    ts = []
    for rep in range(10):
        tr.zero_()
        at.select(x, k, engine=6, cluster_size=4, trace=tr)
        torch.cuda.synchronize()
        t = tr[:64].view(4, 16).cpu().numpy()
        ts.append((t[0, 14] - t[0, 0]) / 1e3)
    print(f"batch {batch} rows sequentially in one cluster: kernel {np.median(ts[3:]):.2f} us -> {np.median(ts[3:]) / batch:.2f} us/row")
