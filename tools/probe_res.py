import sys; sys.path.insert(0, '/root/repo')
import numpy as np, torch, paper_conf_sc_zhangnlw23_b200 as at
n = 1 << 17
for batch in (1, 2, 3):
    for k in (1, 5000):
        x = torch.full((batch, n), 1.0, device="cuda")
        try:
            at.select(x, k, engine=6); torch.cuda.synchronize(); print(batch, k, "ok", at.describe(torch.float32, batch, n, k, engine=6))
        except Exception as e:
            print(batch, k, "ERR", e, at.describe(torch.float32, batch, n, k, engine=6))
