"""GPU tests of the multi-GPU building blocks through the C ABI, on one GPU (several "ranks"
simulated as shards of one row): airtopk_select_shard (global indices, pads for short shards)
written into slots of the gather buffers, then airtopk_select_with_idx — the result must equal the
oracle's single-row top-K of the whole row. Plus the device status word
(duplicate in_idx values are reported, not silently truncated) and argument checks."""
import numpy as np
import pytest

import gen
import oracle
from helpers import BITS_NP, assert_parity, to_bits, to_device

pytestmark = pytest.mark.gpu


def _split_select(raw, dtn, k, world, select_min=True, bounds=None):
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    n = raw.size
    if bounds is None:
        bounds = np.linspace(0, n, world + 1).astype(np.int64)
    x = to_device(raw, dtn).reshape(-1)
    gv = torch.empty(world * k, dtype=x.dtype, device="cuda")
    gi = torch.empty(world * k, dtype=torch.int64, device="cuda")
    for r in range(world):
        lo, hi = int(bounds[r]), int(bounds[r + 1])
        at.select_shard(x[lo:hi].contiguous(), k, lo, n + r * k, largest=not select_min,
                        out=(gv[r * k:(r + 1) * k], gi[r * k:(r + 1) * k]))
    v, i = at.select_with_idx(gv, gi, k, at.merge_idx_bits(n, world, k), largest=not select_min, check=True)
    torch.cuda.synchronize()
    return to_bits(v, dtn), i.cpu().numpy()


@pytest.mark.parametrize("dtn", ["f32", "f16", "bf16", "f64", "u32"])
@pytest.mark.parametrize("select_min", [True, False])
def test_split_row_equals_single_row(dtn, select_min):
    n, k = 3 * (1 << 18) + 12345, 4000
    if dtn == "u32":
        raw = gen.u32(21, n)
    elif dtn == "f64":
        raw = gen.uniform_f64(21, n).view(np.uint64)
    else:
        f = gen.normal_f32(21, n)
        raw = {"f32": f.view(np.uint32), "f16": f.astype(np.float16).view(np.uint16),
               "bf16": (f.view(np.uint32) >> 16).astype(np.uint16)}[dtn]
    for world in (2, 3, 8):
        gv, gi = _split_select(raw, dtn, k, world, select_min)
        assert_parity(raw, dtn, k, select_min, gv, gi)


def test_split_row_ties_across_shards():
    """Heavy ties straddling K across every shard boundary: the lowest GLOBAL indices win."""
    n, k = 1 << 20, 50_000
    raw = gen.adversarial_f32(22, n, m_bits=26).view(np.uint32)  # 64 values, ~16K ties each
    for world in (2, 4, 8):
        gv, gi = _split_select(raw, "f32", k, world)
        assert_parity(raw, "f32", k, True, gv, gi)


@pytest.mark.parametrize("select_min", [True, False])
def test_split_row_shards_shorter_than_k(select_min):
    """Every shard shorter than K: the pad entries (sort last) must never be selected."""
    n, k = 3000, 1200
    raw = gen.uniform_f32(23, n).view(np.uint32)
    gv, gi = _split_select(raw, "f32", k, 4, select_min)        # 750 per shard < 1200
    assert_parity(raw, "f32", k, select_min, gv, gi)
    bounds = np.array([0, 100, 2900, 2950, 3000])               # ragged shards
    gv, gi = _split_select(raw, "f32", k, 4, select_min, bounds=bounds)
    assert_parity(raw, "f32", k, select_min, gv, gi)


def test_shard_outputs_global_indices_and_pads():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    raw = gen.uniform_f32(24, 1000)
    x = torch.from_numpy(raw).cuda()
    v, i = at.select_shard(x, 1500, 7_000_000, 123_456_789)
    torch.cuda.synchronize()
    ii = i.cpu().numpy()
    assert np.array_equal(np.sort(ii[:1000]), 7_000_000 + np.arange(1000))
    assert np.array_equal(ii[1000:], 123_456_789 + np.arange(500))
    assert np.all(v.cpu().numpy()[1000:].view(np.uint32) == 0x7FFFFFFF)   # +NaN, full payload: sorts last


def test_status_reports_duplicate_in_idx():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = torch.from_numpy(gen.adversarial_f32(25, 10_000, m_bits=31)).cuda()   # 2 distinct values
    idx = torch.arange(10_000, device="cuda") % 100                          # duplicate index values
    with pytest.raises(at.DeviceError):
        at.select_with_idx(x, idx, 5000, 20, check=True)
    ok = torch.arange(10_000, device="cuda")
    at.select_with_idx(x, ok, 5000, 20, check=True)


def test_status_clean_on_every_engine():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    for shape, k, kw in (((1, 1 << 16), 32, {}), ((3, 1 << 20), 1000, {}), ((1, 1 << 22), 1 << 12, {"window": -1}),
                         ((100, 1 << 14), 256, {})):
        x = torch.from_numpy(gen.normal_f32(26, shape[0] * shape[1]).reshape(shape)).cuda()
        st = torch.zeros(1, dtype=torch.int32, device="cuda")
        at.select(x, k, status=st, **kw)
        torch.cuda.synchronize()
        assert int(st.item()) == 0


def test_out_and_workspace_checks():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = torch.zeros((2, 1000), device="cuda")
    bad = [(torch.empty((2, 9), device="cuda"), torch.empty((2, 10), dtype=torch.int64, device="cuda")),
           (torch.empty((2, 10), device="cuda"), torch.empty((2, 10), dtype=torch.int32, device="cuda")),
           (torch.empty((2, 10)), torch.empty((2, 10), dtype=torch.int64)),
           (torch.empty((10, 2), device="cuda").t(), torch.empty((2, 10), dtype=torch.int64, device="cuda"))]
    for out in bad:
        with pytest.raises(ValueError):
            at.select(x, 10, out=out)
    with pytest.raises(ValueError):
        at.select(x, 10, workspace=torch.empty(16, dtype=torch.uint8, device="cuda"))
    with pytest.raises(ValueError):
        at.select(x, 10, workspace=torch.empty(1 << 20, dtype=torch.float32, device="cuda"))


@pytest.mark.parametrize("engine,shape,k", [(2, (1, 1 << 17), 32), (5, (8, 1 << 18), 64), (6, (1, 1 << 16), 32)])
def test_debug_timing_bounded_by_trace_len(engine, shape, k):
    """Engines that write per-CTA debug stamps into the trace buffer never write past the buffer the
    caller passed (options.trace_len; the cluster engine's stamps could overrun it)."""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = torch.from_numpy(gen.uniform_f32(41, shape[0] * shape[1]).reshape(shape)).cuda()
    kw = {"cluster_size": 16} if engine == 2 else {}
    big = torch.zeros(1 << 16, dtype=torch.int64, device="cuda")
    at.select(x, k, engine=engine, trace=big[:24], **kw)
    torch.cuda.synchronize()
    assert int(torch.count_nonzero(big[24:]).item()) == 0
    v, i = at.select(x, k, engine=engine, trace=big, **kw)
    torch.cuda.synchronize()
    assert int(torch.count_nonzero(big).item()) > 0   # stamps are written when they fit
    rv, ri = oracle.topk_nth(x.cpu().numpy(), k)
    assert np.array_equal(np.sort(i.cpu().numpy(), axis=1), np.sort(ri, axis=1))


def test_select_on_non_current_device():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs")
    raw = gen.uniform_f32(27, 1 << 20)
    torch.cuda.set_device(0)
    x = torch.from_numpy(raw).to("cuda:1")
    v, i = at.select(x, 1000)
    torch.cuda.synchronize(1)
    assert_parity(raw.view(np.uint32), "f32", 1000, True, v.view(torch.int32).cpu().numpy().view(np.uint32),
                  i.cpu().numpy())


@pytest.mark.parametrize("engine", [0, 1, 2, 5, 6])
def test_sorted_output_option(engine):
    """sorted=True: each row in selection order (keys ascending for select-min / descending for
    select-max, equal keys by ascending index), identical set to the oracle."""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    batch, n, k = 40, 1 << 17, 3000
    raw = gen.adversarial_f32(81, batch * n, m_bits=22).reshape(batch, n)
    x = torch.from_numpy(raw).cuda()
    for largest in (False, True):
        try:
            v, i = at.select(x, k, largest=largest, engine=engine, sorted=True)
        except at.AirTopKError:
            assert engine in (5, 6)  # shape not eligible for that engine
            continue
        torch.cuda.synchronize()
        vb, ii = v.cpu().numpy(), i.cpu().numpy()
        assert_parity(raw.view(np.uint32), "f32", k, not largest, vb.view(np.uint32), ii)
        rv, ri = oracle.topk_sort(raw, k, select_min=not largest)   # canonical (code, index) order
        assert np.array_equal(ii, ri) and np.array_equal(vb.view(np.uint32), rv.view(np.uint32))
    with pytest.raises(at.AirTopKError):
        at.select(x, 4097, sorted=True)
