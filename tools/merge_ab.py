"""Engines for the split-row merge (airtopk_select_with_idx over world x K gathered candidates)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for world, k in ((8, 1 << 16), (2, 1 << 12), (8, 1 << 20)):
    m = world * k
    gv = torch.from_numpy(gen.uniform_f32(99, m) * np.float32(2.0 ** -14)).cuda()
    r = torch.arange(m, device="cuda")
    gi = (r // k) * (1 << 30) + (r % k) * 7
    bits = at.merge_idx_bits(world << 30, world, k)
    for eng in (0, 1, 2):
        try:
            for _ in range(3):
                at.select_with_idx(gv, gi, k, bits, engine=eng)
            torch.cuda.synchronize()
            t = 0.0
            for _ in range(20):
                flush.fill_(1)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                at.select_with_idx(gv, gi, k, bits, engine=eng)
                e1.record()
                e1.synchronize()
                t += e0.elapsed_time(e1)
            print(f"merge world {world} k {k}: engine {eng}: {t / 20 * 1e3:.1f} us", flush=True)
        except Exception as e:  # noqa: BLE001
            print(f"merge world {world} k {k}: engine {eng}: {e}")
