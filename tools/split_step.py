"""One split-row step of 2 shards on one GPU through the C ABI (shard selects into the gather buffers +
merge), for an ncu launch list: every launch must be a libairtopk.so kernel (no torch elementwise
kernels on the path; the NCCL all-gather itself is not part of a single-process run)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_zhangnlw23_b200 as at  # noqa: E402

n, k, world = 1 << 26, 1 << 12, 2
x = torch.from_numpy(gen.uniform_f32(gen.config_seed("c5"), world * n)).cuda()
gv = torch.empty(world * k, dtype=torch.float32, device="cuda")
gi = torch.empty(world * k, dtype=torch.int64, device="cuda")
bits = at.merge_idx_bits(world * n, world, k)
wss = torch.empty(at.lib().airtopk_workspace_bytes_shard(0, n, k), dtype=torch.uint8, device="cuda")
wsm = torch.empty(at.lib().airtopk_workspace_bytes_with_idx(0, world * k, k, bits), dtype=torch.uint8, device="cuda")
out = (torch.empty(k, device="cuda"), torch.empty(k, dtype=torch.int64, device="cuda"))
torch.cuda.synchronize()
for rep in range(2):
    for r in range(world):
        at.select_shard(x[r * n:(r + 1) * n], k, r * n, world * n + r * k, out=(gv[r * k:(r + 1) * k], gi[r * k:(r + 1) * k]),
                        workspace=wss)
    at.select_with_idx(gv, gi, k, bits, workspace=wsm, out=out)
torch.cuda.synchronize()
print("split step done")
