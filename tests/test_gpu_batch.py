"""GPU parity of the batched engine (engine 5, csrc/engine_batch.cuh): one cooperative launch per
batch — sample, single-read window stream into fixed per-chunk slots, per-row finish — plus the
cluster-engine fallback launch for rows whose window failed. Every output is compared with the CPU
oracle (identical value bits, identical index set under the lowest-index rule). White-box checks
read the per-row outcome (RowState.win_state: 4 = finished by the batch kernel, 3 = fallback) from
the workspace so both paths are known to have run."""
import numpy as np
import pytest

import gen
import oracle
from helpers import assert_parity, to_bits, to_device

pytestmark = pytest.mark.gpu

ROWSTATE_BYTES = 128
WIN_STATE_OFF = 88  # RowState: 8 x u64, ticket, npass, stop1, j, error, src1, win_state (csrc/device.cuh)


def _run(raw, dtn, k, select_min=True, engine=5, **kw):
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = to_device(raw, dtn)
    batch, n = x.shape
    need = at.workspace_bytes(x.dtype, batch, n, k, engine=engine)
    ws = torch.zeros(need, dtype=torch.uint8, device="cuda")
    v, i = at.select(x, k, largest=not select_min, engine=engine, workspace=ws, check=True, **kw)
    torch.cuda.synchronize()
    states = ws[: batch * ROWSTATE_BYTES].view(batch, ROWSTATE_BYTES)[:, WIN_STATE_OFF:WIN_STATE_OFF + 4]
    states = states.contiguous().view(torch.int32).reshape(-1).cpu().numpy()
    return to_bits(v, dtn), i.cpu().numpy(), states


def _keys(dtn, dist, seed, n):
    if dtn == "u32":
        return gen.u32(seed, n)
    if dtn == "f64":
        return gen.uniform_f64(seed, n).view(np.uint64)
    f = gen.keys(dist, seed, n)
    return {"f32": f.view(np.uint32), "f16": f.astype(np.float16).view(np.uint16),
            "bf16": (f.view(np.uint32) >> 16).astype(np.uint16)}[dtn]


def test_auto_picks_batch_engine_for_c2():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    d = at.describe(torch.float32, 100, 1 << 20, 256)
    assert d["engine"] == 5 and d["launches"] == 2


@pytest.mark.parametrize("dtn", ["f32", "f16", "bf16", "f64", "u32"])
@pytest.mark.parametrize("select_min", [True, False])
def test_batch_dtypes(dtn, select_min):
    batch, n, k = 37, 1 << 18, 100
    raw = _keys(dtn, "normal", 31, batch * n).reshape(batch, n)
    gv, gi, st = _run(raw, dtn, k, select_min)
    assert_parity(raw, dtn, k, select_min, gv, gi)
    assert np.all(st == 4)


@pytest.mark.parametrize("batch,n,k", [(2, 1 << 14, 1), (7, (1 << 16) + 16, 10), (100, 1 << 20, 256),
                                       (300, 1 << 16, 64), (160, 3 << 16, 512), (5, 1 << 22, 1500),
                                       (3, 1 << 20, 1)])
@pytest.mark.parametrize("dist", ["uniform", "normal"])
def test_batch_shapes(batch, n, k, dist):
    raw = gen.keys(dist, 32, batch * n).reshape(batch, n).view(np.uint32)
    gv, gi, st = _run(raw, "f32", k)
    assert_parity(raw, "f32", k, True, gv, gi)
    assert np.all(st == 4)


def test_batch_ties_and_special_values():
    batch, n, k = 20, 1 << 16, 300
    raw = gen.adversarial_f32(33, batch * n, m_bits=22).reshape(batch, n).view(np.uint32).copy()
    raw[3] = 0x3F800000                       # a row of equal keys: no window -> fallback
    raw[4, ::7] = 0x80000000                  # -0.0 below every positive key
    raw[5, 100:200] = 0x7FC00000              # +NaN (sorts last for select-min)
    raw[6, 1000:1500] = 0xFF800000            # -inf
    for sm in (True, False):
        gv, gi, st = _run(raw, "f32", k, sm)
        assert_parity(raw, "f32", k, sm, gv, gi)
        assert st[3] == 3


def test_batch_slot_overflow_falls_back():
    """A contiguous run of tiny keys floods a few chunk slots: those rows must take the
    fallback launch and still be exact; the other rows finish in the batch kernel."""
    batch, n, k = 16, 1 << 20, 256
    raw = gen.uniform_f32(34, batch * n).reshape(batch, n).copy()
    for r in range(0, batch, 2):
        s = 5000 + 37 * r
        raw[r, s:s + 300] = np.float32(1e-9) * (1 + np.arange(300, dtype=np.float32))
    gv, gi, st = _run(raw.view(np.uint32), "f32", k)
    assert_parity(raw.view(np.uint32), "f32", k, True, gv, gi)
    assert np.all(st[0::2] == 3) and np.all(st[1::2] == 4)


def test_batch_window_miss_falls_back():
    """Keys placed where the stratified sample does not look (white box: runs of 32 at
    run * stride + (stride - 32) / 2) make the window hold fewer than K keys: the window check
    fails, the fallback is exact."""
    batch, n, k = 4, 1 << 20, 4000
    ns = min(max(n // 128, 4096), 16384) // 32 * 32
    stride = n // (ns // 32)
    raw = np.full((batch, n), 0.9, np.float32) + gen.uniform_f32(35, batch * n).reshape(batch, n) * np.float32(0.01)
    pos = (np.arange(ns // 32)[:, None] * stride + (stride - 32) // 2 + np.arange(32)[None, :]).reshape(-1)
    raw[:, pos] = np.float32(0.001) * gen.uniform_f32(36, pos.size)[None, :]
    gv, gi, st = _run(raw.view(np.uint32), "f32", k)
    assert_parity(raw.view(np.uint32), "f32", k, True, gv, gi)
    assert np.all(st == 3)


def test_batch_early_stop_off_and_k_range():
    batch, n = 9, 1 << 17
    raw = gen.normal_f32(37, batch * n).reshape(batch, n).view(np.uint32)
    for k in (1, 2, 33, 255, 1000):
        gv, gi, _ = _run(raw, "f32", k, early_stop=-1)
        assert_parity(raw, "f32", k, True, gv, gi)


def test_batch_engine_rejects_misaligned_or_ineligible():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = torch.zeros(4 * 65536 + 1, device="cuda")[1:].reshape(4, 65536)  # 4-byte offset: not 16-aligned
    with pytest.raises(at.AirTopKError):
        at.select(x, 10, engine=5)
    v, i = at.select(x, 10)  # AUTO picks another engine
    torch.cuda.synchronize()
    assert sorted(i[0].tolist()) == list(range(10))
