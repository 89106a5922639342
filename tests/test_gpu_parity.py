"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, bit-exact.

The bar (BASELINE.json north_star): identical value multiset and identical index set under the
lowest-index tie rule, on seeded synthetic inputs shaped like the paper's workloads (PAPER.md:231,
235-241), plus the edge cases the method has (K = 1, K = N, ties straddling K, early stop,
never/always buffering, misaligned rows, every key type).
"""
import numpy as np
import pytest

import gen
import oracle
from helpers import assert_parity, gpu_select, to_device, to_bits

pytestmark = pytest.mark.gpu


def _keys(dist, seed, batch, n, m=20):
    return gen.keys(dist, seed, batch * n, m_bits=m).reshape(batch, n)


# ---------------------------------------------------------------- the five BASELINE configs

def test_c1_full():
    x = gen.config_keys("c1")
    v, i = gpu_select(x, "f32", 32)
    assert_parity(x, "f32", 32, True, v, i)


def test_c2_full():
    x = gen.config_keys("c2")
    v, i = gpu_select(x, "f32", 256)
    assert_parity(x, "f32", 256, True, v, i)


def test_c4_full_adversarial_ties():
    x = gen.config_keys("c4")
    v, i = gpu_select(x, "f32", 50000)
    # closed form: every result is 1.0f and the indices are the first 50,000
    # positions holding 1.0f
    first = np.flatnonzero(x[0] == np.float32(1.0))[:50000]
    assert np.all(v.view(np.uint32) == 0x3F800000)
    assert np.array_equal(np.sort(i[0]), first)
    assert_parity(x, "f32", 50000, True, v, i)


def test_c3_full():
    x = gen.config_keys("c3")
    v, i = gpu_select(x, "f32", 1 << 20)
    assert_parity(x, "f32", 1 << 20, True, v, i)


def test_c5_shard_full():
    """One 2^30 shard of the c5 row (global indices 2^30 .. 2^31-1) with K = 2^16."""
    n = 1 << 30
    x = gen.uniform_f32(gen.config_seed("c5"), n, offset=n)
    v, i = gpu_select(x, "f32", 1 << 16)
    assert_parity(x, "f32", 1 << 16, True, v, i)


# ---------------------------------------------------------------- distributions x shapes

@pytest.mark.parametrize("dist", ["uniform", "normal", "adversarial"])
@pytest.mark.parametrize("batch,n,k", [(1, 1 << 20, 1), (1, 1 << 20, 1000), (3, 100003, 4097),
                                       (100, 1 << 14, 256), (7, 5000, 5000 - 1), (1, 1 << 22, 1 << 12)])
@pytest.mark.parametrize("select_min", [True, False])
def test_distributions(dist, batch, n, k, select_min):
    x = _keys(dist, 123, batch, n)
    v, i = gpu_select(x, "f32", k, select_min)
    assert_parity(x, "f32", k, select_min, v, i)


@pytest.mark.parametrize("m", [10, 20, 28, 31, 32])
def test_adversarial_prefix_lengths(m):
    x = _keys("adversarial", 9, 2, 1 << 18, m)
    for k in (1, 77, 30000):
        v, i = gpu_select(x, "f32", k)
        assert_parity(x, "f32", k, True, v, i)


# ---------------------------------------------------------------- edge cases

@pytest.mark.parametrize("n", [1, 2, 3, 31, 32, 33, 255, 1000, 4097, 65537])
def test_small_and_ragged(n):
    x = gen.uniform_f32(5, n)
    for k in sorted({1, max(1, n // 2), max(1, n - 1), n}):
        v, i = gpu_select(x, "f32", k)
        assert_parity(x, "f32", k, True, v, i)


@pytest.mark.parametrize("off", [1, 2, 3])
def test_misaligned_rows(off):
    x = _keys("normal", 4, 3, 7777)
    v, i = gpu_select(x, "f32", 100, offset_elems=off)
    assert_parity(x, "f32", 100, True, v, i)


def test_all_equal_and_two_valued():
    x = np.full((2, 100000), 2.5, np.float32)
    v, i = gpu_select(x, "f32", 1234)
    assert np.array_equal(np.sort(i, axis=1), np.tile(np.arange(1234), (2, 1)))
    y = np.where(gen.u32(1, 300000) & 1, np.float32(1), np.float32(2)).astype(np.float32)
    for k in (1, 1000, 150000, 200000):
        v, i = gpu_select(y, "f32", k)
        assert_parity(y, "f32", k, True, v, i)


def test_special_values():
    bits = gen.u32(77, 200000)
    pool = np.array([0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000, 0xFFC00001, 0x00000001,
                     0x80000001, 0x7F7FFFFF, 0xFF7FFFFF, 0x3F800000, 0xBF800000], np.uint32)
    raw = np.where(bits % 3 == 0, pool[bits % pool.size], bits)
    for k in (1, 13, 5000, 199999):
        for sm in (True, False):
            v, i = gpu_select(raw, "f32", k, sm)
            assert_parity(raw, "f32", k, sm, v, i)


@pytest.mark.parametrize("dtn", ["f16", "bf16", "f64", "u32"])
@pytest.mark.parametrize("pool", [0, 5])
def test_other_dtypes(dtn, pool):
    n = 300001
    u = gen.u64(31, n)
    if pool:
        u = gen.u64(32, pool)[u % np.uint64(pool)]
    raw = u.astype({"f16": np.uint16, "bf16": np.uint16, "f64": np.uint64, "u32": np.uint32}[dtn])
    for k in (1, 999, 150000):
        for sm in (True, False):
            v, i = gpu_select(raw, dtn, k, sm)
            assert_parity(raw, dtn, k, sm, v, i)


def test_f16_exhaustive():
    raw = np.arange(1 << 16, dtype=np.uint32).astype(np.uint16)
    raw = raw[np.argsort(gen.u32(3, 1 << 16))]
    for k in (1, 1024, 40000, 65535):
        v, i = gpu_select(raw, "f16", k)
        assert_parity(raw, "f16", k, True, v, i)


# ---------------------------------------------------------------- adaptive strategy / engine knobs

@pytest.mark.parametrize("alpha", [1, 4, 128, 1 << 40])
@pytest.mark.parametrize("dist,m", [("uniform", 20), ("adversarial", 20), ("adversarial", 10)])
def test_alpha_invariance(alpha, dist, m):
    """Results are independent of alpha: always / default / never buffering."""
    x = _keys(dist, 21, 2, 1 << 20, m)
    for k in (5, 3000):
        v, i = gpu_select(x, "f32", k, alpha=alpha)
        assert_parity(x, "f32", k, True, v, i)


@pytest.mark.parametrize("cpr", [1, 2, 7, 300])
def test_ctas_per_row(cpr):
    x = _keys("uniform", 8, 3, 200000)
    v, i = gpu_select(x, "f32", 500, ctas_per_row=cpr)
    assert_parity(x, "f32", 500, True, v, i)


# ---------------------------------------------------------------- per-pass state vs the oracle's Algorithm 1 trace

@pytest.mark.parametrize("dist,m,k,alpha", [("uniform", 20, 1000, 128), ("normal", 20, 77, 128),
                                            ("adversarial", 20, 5000, 128), ("adversarial", 10, 100, 4),
                                            ("uniform", 20, 1 << 12, 1 << 40)])
def test_trace_matches_algorithm1(dist, m, k, alpha):
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    n = 1 << 20
    x = gen.keys(dist, 55, n, m_bits=m)
    tr = at.trace_buffer(1)
    xd = to_device(x, "f32").reshape(1, -1)
    at.select(xd, k, alpha=alpha, trace=tr, engine=at.ENGINE_GRID, window=-1)  # the paper's passes
    torch.cuda.synchronize()
    g = tr.cpu().numpy()[0]
    codes = oracle.codes(x)
    _, recs, _ = oracle.radix_trace(codes, k, r_bits=32, b=11, idx_bits=20, alpha=alpha)
    emitted = 0
    for q, r in enumerate(recs[:-1]):
        t = dict(zip(at._lib.TRACE_FIELDS, g[q].tolist()))
        emitted += r["emitted"]
        for f in ("width", "src_L", "stored", "j", "K", "C", "Cp", "early_stop", "read"):
            assert t[f] == r[f], f"pass {q} field {f}: gpu {t[f]} oracle {r[f]}"
        assert t["emitted"] == emitted
    assert g[len(recs) - 1][0] == -1      # no scan after the early stop


# ---------------------------------------------------------------- other entry points

def test_with_idx_merge():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    n, k = 200000, 5000
    x = gen.adversarial_f32(3, n, m_bits=24)
    perm = np.argsort(gen.u32(4, n)).astype(np.int64)
    gid = perm * 3 + 1000                       # distinct, not position-ordered
    v, i = at.select_with_idx(to_device(x, "f32"), torch.from_numpy(gid).cuda(), k, idx_bits=21)
    rv, ri = oracle.topk_with_idx(x, gid, k)
    gi = i.cpu().numpy()
    assert np.array_equal(np.sort(gi), np.sort(ri))
    inv = np.full(gid.max() + 1, -1, np.int64)
    inv[gid] = np.arange(n)
    assert np.array_equal(to_bits(v, "f32"), x[inv[gi]].view(np.uint32))


def test_select_host_e2e():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = gen.config_keys("c2", batch=10)
    xt = torch.from_numpy(x).pin_memory()
    v, i = at.select_host(xt, 256)
    assert_parity(x, "f32", 256, True, v.numpy().view(np.uint32), i.numpy())


def test_typed_entry_points_pool_workspace():
    import ctypes
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = gen.config_keys("c1")
    xd = to_device(x, "f32")
    v = torch.empty((1, 32), dtype=torch.float32, device="cuda")
    i = torch.empty((1, 32), dtype=torch.int64, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    assert at.lib().airtopk_select_f32(xd.data_ptr(), 1, x.shape[1], 32, 1, v.data_ptr(), i.data_ptr(), s) == 0
    torch.cuda.synchronize()
    assert_parity(x, "f32", 32, True, to_bits(v, "f32"), i.cpu().numpy())


def test_repeated_calls_reuse_workspace():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    x = _keys("normal", 70, 4, 1 << 16)
    xd = to_device(x, "f32")
    ws = torch.empty(at.workspace_bytes(torch.float32, 4, 1 << 16, 300), dtype=torch.uint8, device="cuda")
    for _ in range(3):
        v, i = at.select(xd, 300, workspace=ws)
    torch.cuda.synchronize()
    assert_parity(x, "f32", 300, True, to_bits(v, "f32"), i.cpu().numpy())


# ---------------------------------------------------------------- both engines, every cluster size

@pytest.mark.parametrize("engine,cs", [(1, 0), (2, 1), (2, 2), (2, 4), (2, 8), (2, 16)])
@pytest.mark.parametrize("dist,batch,n,k", [("normal", 37, 1 << 16, 256), ("uniform", 3, 300001, 5000),
                                            ("adversarial", 5, 1 << 18, 20000), ("uniform", 1, 1 << 16, 32)])
def test_engines(engine, cs, dist, batch, n, k):
    x = _keys(dist, 61, batch, n)
    for sm in (True, False):
        v, i = gpu_select(x, "f32", k, sm, engine=engine, cluster_size=cs)
        assert_parity(x, "f32", k, sm, v, i)


@pytest.mark.parametrize("dtn", ["f16", "bf16", "f64", "u32"])
def test_cluster_engine_dtypes(dtn):
    u = gen.u64(91, 8 * 20011)
    raw = u.astype({"f16": np.uint16, "bf16": np.uint16, "f64": np.uint64, "u32": np.uint32}[dtn]).reshape(8, 20011)
    for k in (1, 500, 20010):
        v, i = gpu_select(raw, dtn, k, True, engine=2)
        assert_parity(raw, dtn, k, True, v, i)


@pytest.mark.parametrize("alpha", [1, 128, 1 << 40])
def test_cluster_engine_alpha(alpha):
    x = _keys("adversarial", 13, 6, 1 << 17, 10)
    v, i = gpu_select(x, "f32", 3000, alpha=alpha, engine=2)
    assert_parity(x, "f32", 3000, True, v, i)


# ---------------------------------------------------------------- sample-guided window (NEXT #1)

def _sample_positions(n):
    """The positions the sample kernel reads (runs of 32 at stratified offsets, see api.cu)."""
    ns = min(max(n // 128, 4096), 16384)
    ns = min(ns, n // 2) // 32 * 32
    runs = ns // 32
    stride = n // runs
    base = np.arange(runs, dtype=np.int64) * stride + (stride - 32) // 2
    return (base[:, None] + np.arange(32)[None, :]).reshape(-1)


@pytest.mark.parametrize("window", [-1, 1])
@pytest.mark.parametrize("dist,m", [("uniform", 20), ("normal", 20), ("adversarial", 20), ("adversarial", 12)])
@pytest.mark.parametrize("k", [1, 100, 77777, 1 << 19])
def test_window_on_off(window, dist, m, k):
    x = _keys(dist, 71, 2, 1 << 20, m)
    for sm in (True, False):
        v, i = gpu_select(x, "f32", k, sm, window=window, engine=1)
        assert_parity(x, "f32", k, sm, v, i)


@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("case", ["high", "low", "ties"])
def test_window_fallback(case, engine):
    """Inputs built so the stratified sample misrepresents the row: the window pass must detect the
    miss (R >= K or K > R + W) and fall back to the paper's passes, exactly."""
    n = 1 << 20
    x = gen.uniform_f32(8, n)
    pos = _sample_positions(n)
    if case == "high":
        x[pos] = np.float32(1e30)
        ks = (1000, 500000)
    elif case == "low":
        x[pos] = np.float32(-1e30)
        ks = (len(pos) + 5, 500000)
    else:
        x[:] = np.float32(3.0)
        x[pos] = np.float32(2.0)
        ks = (1, len(pos) + 1, 700000)
    for k in ks:
        v, i = gpu_select(x, "f32", k, True, window=1, engine=engine)
        assert_parity(x, "f32", k, True, v, i)


@pytest.mark.parametrize("dist,batch,n,k", [("normal", 100, 1 << 20, 256), ("adversarial", 3, 1 << 22, 5000),
                                            ("uniform", 7, 1 << 19, 1), ("uniform", 2, 1 << 21, 20000)])
@pytest.mark.parametrize("cluster_tail", [False, True])
def test_window_tail(dist, batch, n, k, cluster_tail, monkeypatch):
    """grid engine window pass (window=1: AUTO sends batches to the batched engine) followed by the
    grid passes, or — opt-in, AIRTOPK_CLUSTER_TAIL=1 — by one cluster-engine launch finishing
    every row (tail mode)"""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    if cluster_tail:
        monkeypatch.setenv("AIRTOPK_CLUSTER_TAIL", "1")
        assert at.describe(torch.float32, batch, n, k, window=1)["launches"] == 3
    x = _keys(dist, 33, batch, n)
    for sm in (True, False):
        v, i = gpu_select(x, "f32", k, sm, window=1)
        assert_parity(x, "f32", k, sm, v, i)


def test_cluster_tail_off_by_default_and_miss_safe():
    """AUTO never picks the cluster tail (a rejected window restarted the row inside
    one cluster); a constant row with a tiny K — the window is rejected — runs on the grid and stays
    exact"""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    n = 1 << 26
    d = at.describe(torch.float32, 1, n, 10)
    assert d["engine"] == 1 and d["cluster_size"] == 0
    x = np.full((1, n), 0.5, np.float32)
    v, i = gpu_select(x, "f32", 10, True)
    assert_parity(x, "f32", 10, True, v, i)


def test_window_describe():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    d = at.describe(torch.float32, 1, 1 << 30, 1 << 20)
    assert d["engine"] == 1 and d["launches"] == 3   # sample, window pass, fused tail (every other pass)
    d = at.describe(torch.float32, 1, 1 << 30, 1 << 20, window=-1)
    assert d["launches"] == d["passes"] + 1


# ---------------------------------------------------------------- bulk-copy (TMA) streaming vs register loads

@pytest.mark.parametrize("tma", [-1, 1])
@pytest.mark.parametrize("window", [-1, 1])
@pytest.mark.parametrize("dist,m,batch,n,k,off", [("uniform", 20, 1, (1 << 22) + 77, 3000, 0),
                                                  ("adversarial", 20, 2, 1 << 22, 40000, 1),
                                                  ("normal", 20, 3, 999999, 17, 3),
                                                  ("adversarial", 12, 1, 1 << 21, 1 << 20, 2)])
def test_tma_streaming(tma, window, dist, m, batch, n, k, off):
    x = _keys(dist, 44, batch, n, m)
    for sm in (True, False):
        v, i = gpu_select(x, "f32", k, sm, offset_elems=off, tma=tma, window=window, engine=1)
        assert_parity(x, "f32", k, sm, v, i)


# ---------------------------------------------------------------- rows longer than 2^32 (64-bit indices)

@pytest.mark.parametrize("dtn,largest", [("f16", False), ("f32", False), ("f16", True)])
def test_row_longer_than_2p32(dtn, largest):
    """len = 2^32 + 2^20 + 3 (the u64-index path, include/airtopk.h "Limits"; the c5 row
    on one GPU). Every key equals v0 except planted keys at positions on both sides of 2^32, some
    equal to each other and some equal to v0's neighbours. Property that holds at any size: the
    top-K of such a row = the top-K of the sub-row made of the planted positions plus the K lowest
    non-planted positions (all v0), kept in index order, since every other element is a v0 with a
    higher index (P:78 with the lowest-index rule). That sub-row goes to the CPU oracle."""
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    n = (1 << 32) + (1 << 20) + 3
    k = 97
    npdt = {"f16": np.float16, "f32": np.float32}[dtn]
    tdt = {"f16": torch.float16, "f32": torch.float32}[dtn]
    rng = np.random.default_rng(4321)
    pos = np.unique(np.concatenate([
        rng.integers(0, 1 << 32, 40), rng.integers(1 << 32, n, 40),
        [0, 5, (1 << 32) - 1, 1 << 32, (1 << 32) + 1, n - 1]]).astype(np.int64))
    vals = rng.choice(np.array([0.25, 0.5, 0.75, 1.0, 1.5, 2.0, -3.0, 7.0], dtype=npdt), pos.size)
    v0 = npdt(1.0)
    x = torch.full((n,), float(v0), dtype=tdt, device="cuda")
    x[torch.from_numpy(pos).cuda()] = torch.from_numpy(vals).cuda()
    v, i = at.select(x.reshape(1, n), k, largest=largest)
    torch.cuda.synchronize()
    # the sub-row: planted positions + the k lowest positions holding v0 that were not planted
    fill = np.setdiff1d(np.arange(k + pos.size, dtype=np.int64), pos)[:k]
    sub_pos = np.concatenate([pos, fill])
    order = np.argsort(sub_pos)
    sub_pos = sub_pos[order]
    sub_val = np.concatenate([vals, np.full(fill.size, v0, npdt)])[order]
    bits = {"f16": np.uint16, "f32": np.uint32}[dtn]
    rv, ri = oracle.topk_nth(sub_val.view(bits)[None, :], k, not largest, dt=oracle.DT_NAMES[dtn])
    gi = np.sort(i.cpu().numpy()[0])
    assert gi.max() >= 0
    assert np.array_equal(gi, np.sort(sub_pos[ri[0]])), "index set differs (64-bit index path)"
    gv = to_bits(v, dtn)[0]
    assert np.array_equal(np.sort(gv), np.sort(rv[0].view(bits)))
    del x
    torch.cuda.empty_cache()


# ---------------------------------------------------------------- GridSelect (NEXT #3)

@pytest.mark.parametrize("dist,m", [("uniform", 20), ("normal", 20), ("adversarial", 20), ("adversarial", 28)])
@pytest.mark.parametrize("batch,n,k", [(1, 1 << 16, 32), (1, 1 << 16, 1), (3, 100003, 256), (5, 1000, 100),
                                       (2, 33, 33), (4, 31, 7), (1, 1 << 20, 200), (1, 1 << 20, 2048),
                                       (2, 300001, 1500), (3, 5000, 1024)])
@pytest.mark.parametrize("select_min", [True, False])
@pytest.mark.parametrize("engine", [4, 7])
def test_gridselect(dist, m, batch, n, k, select_min, engine):
    """GridSelect with the shared queue (engine 4) and the per-thread-queue variant (engine 7, the
    Fig. 11 ablation), K up to the paper's 2048."""
    x = _keys(dist, 131, batch, n, m=m)
    v, i = gpu_select(x, "f32", k, select_min, engine=engine)
    assert_parity(x, "f32", k, select_min, v, i)


def test_gridselect_rejects_k_above_2048():
    import torch
    import paper_conf_sc_zhangnlw23_b200 as at
    with pytest.raises(at.AirTopKError):
        at.select(torch.zeros((1, 5000), device="cuda"), 2049, engine=4)


@pytest.mark.parametrize("dtn", ["f16", "bf16", "u32"])
def test_gridselect_dtypes(dtn):
    u = gen.u64(92, 6 * 20011)
    raw = u.astype({"f16": np.uint16, "bf16": np.uint16, "u32": np.uint32}[dtn]).reshape(6, 20011)
    for k in (1, 64, 256, 2048):
        for sm in (True, False):
            v, i = gpu_select(raw, dtn, k, sm, engine=4)
            assert_parity(raw, dtn, k, sm, v, i)


def test_gridselect_sorted_output_and_c1():
    """GridSelect returns each row sorted in the selection order (composite key, lowest index first
    among equal keys), on the c1 workload."""
    x = gen.config_keys("c1")
    v, i = gpu_select(x, "f32", 32, True, engine=4)
    assert_parity(x, "f32", 32, True, v, i)
    vals = v.reshape(-1).view(np.float32).astype(np.float64)
    idx = i.reshape(-1)
    for a in range(31):
        assert vals[a] < vals[a + 1] or (vals[a] == vals[a + 1] and idx[a] < idx[a + 1])


@pytest.mark.parametrize("dtn", ["f16", "bf16", "f64", "u32"])
def test_other_dtypes_concentrated(dtn):
    """Keys sharing long leading bit prefixes (c4-like adversarial M=20 values converted to each key
    type) through the window path: window digit skips, member-extreme skips, mass ties."""
    x = gen.adversarial_f32(77, 1 << 20, m_bits=20)
    if dtn == "f64":
        raw = x.astype(np.float64).view(np.uint64)
    elif dtn == "f16":
        raw = x.astype(np.float16).view(np.uint16)
    elif dtn == "bf16":
        raw = (x.view(np.uint32) >> 16).astype(np.uint16)  # truncation: the top 16 bits
    else:
        raw = x.view(np.uint32)
    raw = raw.reshape(1, -1)
    for k in (1, 1000, 50000):
        for sm in (True, False):
            v, i = gpu_select(raw, dtn, k, sm)
            assert_parity(raw, dtn, k, sm, v, i)


@pytest.mark.parametrize("engine", [0, 1, 2])
@pytest.mark.parametrize("dist,batch,n,k", [("uniform", 1, 1 << 20, 1000), ("normal", 7, 1 << 16, 256),
                                            ("adversarial", 1, 1 << 20, 5000)])
def test_early_stop_off_invariance(engine, dist, batch, n, k):
    """Early stopping only skips work: with it disabled (the Fig. 10 ablation) every
    engine returns the same exact result, for the paper's passes and the window path."""
    x = _keys(dist, 151, batch, n)
    for window in (-1, 0):
        if engine == 2 and window == 0:
            continue
        v, i = gpu_select(x, "f32", k, True, engine=engine, window=window, early_stop=-1)
        assert_parity(x, "f32", k, True, v, i)


@pytest.mark.parametrize("dtn", ["f16", "bf16"])
@pytest.mark.parametrize("front", [False, True])
@pytest.mark.parametrize("select_min", [True, False])
def test_window_16bit_extreme_codes(dtn, front, select_min):
    """Regression (found by tests/fuzz_gpu.py): 16-bit keys whose selected code is the extreme one
    (-NaN with full payload for select-min: code 0), ties partly in the scalar tail of a row whose
    length is not a multiple of 8, through the window pass. The raw-bit window test must widen the
    16-bit all-ones mask without integer promotion."""
    n = 1510669
    raw = np.sort(gen.u64(5, n).astype(np.uint16))
    if not select_min:
        raw = raw[::-1].copy()
    if front:
        cnt = int((raw == raw[-1]).sum())
        raw = np.concatenate([raw[-cnt:], raw[:-cnt]])
    raw = raw.reshape(1, n)
    for k in (1, 2, 17):
        for window in (0, 1):
            v, i = gpu_select(raw, dtn, k, select_min, window=window)
            assert_parity(raw, dtn, k, select_min, v, i)
