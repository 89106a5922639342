"""The paper's kernel-organisation ablations (airtopk_select_ablation, csrc/ablation.cu):
naive four-kernels-per-iteration (Fig. 2), iteration-fused (Fig. 3), fused last filter, with b = 8
and b = 11 — every variant must return exactly the oracle's set, and launch the number of kernels
the paper counts."""
import numpy as np
import pytest

import gen
from helpers import assert_parity, to_bits

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("design", [0, 1, 2])
@pytest.mark.parametrize("b", [8, 11])
@pytest.mark.parametrize("dist,batch,n,k", [("uniform", 1, 1 << 20, 2048), ("normal", 3, 100003, 777),
                                            ("adversarial", 2, 1 << 18, 5000), ("uniform", 1, 1000, 1)])
def test_ablation_parity(design, b, dist, batch, n, k):
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    raw = gen.keys(dist, 71, batch * n, m_bits=20).reshape(batch, n)
    x = torch.from_numpy(raw).cuda()
    for largest in (False, True):
        v, i, nk = at.select_ablation(x, k, design, b, largest=largest)
        torch.cuda.synchronize()
        assert_parity(raw.view(np.uint32), "f32", k, not largest, to_bits(v, "f32"), i.cpu().numpy())


def test_ablation_kernel_counts():
    """naive b=8 on 32-bit keys: 4 iterations x 4 kernels = 16 (Fig. 2) over the code digits;
    fused b=11: 3 iteration-fused kernels + 1 last filter = 4; index digits add passes."""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = torch.from_numpy(gen.uniform_f32(72, 1 << 12)).cuda()   # 12 index bits: 2 index digits at b=8
    _, _, nk = at.select_ablation(x, 10, 0, 8)
    assert nk == 4 * (4 + 2)
    _, _, nk = at.select_ablation(x, 10, 1, 11)
    assert nk == (3 + 2) + 1
    _, _, nk = at.select_ablation(x, 10, 2, 11)
    assert nk == 3 + 2
