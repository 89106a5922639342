"""GPU parity of the resident-cluster engine (engine 6, csrc/engine_resident.cuh): rows held in
shared memory as codes, one cluster barrier per radix pass, small finish in CTA 0. Compared with the
CPU oracle element by element (value bits, index set under the lowest-index rule)."""
import numpy as np
import pytest

import gen
from helpers import assert_parity, gpu_select

pytestmark = pytest.mark.gpu


def _keys(dtn, dist, seed, n):
    if dtn == "u32":
        return gen.u32(seed, n)
    if dtn == "f64":
        return gen.uniform_f64(seed, n).view(np.uint64)
    f = gen.keys(dist, seed, n, m_bits=24)
    return {"f32": f.view(np.uint32), "f16": f.astype(np.float16).view(np.uint16),
            "bf16": (f.view(np.uint32) >> 16).astype(np.uint16)}[dtn]


def test_auto_picks_resident_for_c1():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    d = at.describe(torch.float32, 1, 1 << 16, 32)
    assert d["engine"] == 6 and d["launches"] == 1


@pytest.mark.parametrize("dtn", ["f32", "f16", "bf16", "f64", "u32"])
@pytest.mark.parametrize("dist", ["uniform", "normal", "adversarial"])
@pytest.mark.parametrize("select_min", [True, False])
def test_resident_dtypes(dtn, dist, select_min):
    batch, n, k = 3, (1 << 16) + 24, 300
    raw = _keys(dtn, dist, 41, batch * n).reshape(batch, n)
    gv, gi = gpu_select(raw, dtn, k, select_min, engine=6)
    assert_parity(raw, dtn, k, select_min, gv, gi)


@pytest.mark.parametrize("batch,n,k", [(1, 1 << 16, 32), (1, 1000, 10), (1, 2, 1), (4, 5000, 4999),
                                       (1, 1 << 19, 1000), (1, (1 << 19) - 5, 3), (20, (1 << 15) + 3, 7),
                                       (500, 4096, 64), (2, 1 << 18, 70000)])
def test_resident_shapes(batch, n, k):
    raw = gen.uniform_f32(42, batch * n).reshape(batch, n).view(np.uint32)
    gv, gi = gpu_select(raw, "f32", k, True, engine=6)
    assert_parity(raw, "f32", k, True, gv, gi)


@pytest.mark.parametrize("cs", [1, 2, 4, 8, 16])
def test_resident_cluster_sizes(cs):
    n, k = 30000, 777
    raw = gen.normal_f32(43, 2 * n).reshape(2, n).view(np.uint32)
    gv, gi = gpu_select(raw, "f32", k, True, engine=6, cluster_size=cs)
    assert_parity(raw, "f32", k, True, gv, gi)


def test_resident_ties_index_digits_and_specials():
    n = 1 << 17
    raw = np.full((3, n), 0x3F800000, np.uint32)             # all equal: index digits decide
    raw[1, ::3] = 0x3F000000
    raw[2, 5:50] = 0x7FC00000                                  # +NaN
    raw[2, 60:70] = 0x80000000                                 # -0.0
    for k in (1, 5000, 43690, n - 1):
        for sm in (True, False):
            gv, gi = gpu_select(raw, "f32", k, sm, engine=6)
            assert_parity(raw, "f32", k, sm, gv, gi)


def test_resident_early_stop_off_and_misaligned():
    n = 40000
    raw = gen.normal_f32(44, 2 * n + 1).view(np.uint32)
    x = raw[1:].reshape(2, n)
    for k in (1, 33, 3000):
        gv, gi = gpu_select(x, "f32", k, True, engine=6, early_stop=-1, offset_elems=1)
        assert_parity(x, "f32", k, True, gv, gi)
