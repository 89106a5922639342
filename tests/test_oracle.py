"""Pins of the CPU oracle against things other than itself (CPU only).

Each test names what pins it: the problem definition, a library routine that
reduces to the same result (numpy stable argsort), exhaustive enumeration, closed forms on
adversarial inputs, the Figure 1 worked example, and
the paper's own statements about Algorithm 1.
"""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------------------------------------
# helpers (test-side, independent of the oracle's arithmetic)

def f16_all():
    return np.arange(1 << 16, dtype=np.uint32).astype(np.uint16)


def check_definition_f(x, vals, idx, k, select_min=True):
    """PAPER.md:78 constraints on floats without NaN: L[I[i]] = V[i] bitwise, |I| = K distinct,
    V[i] <= L[j] (>= for select-max) for every j not in I."""
    x = np.asarray(x)
    assert idx.shape == (k,) and len(set(idx.tolist())) == k
    assert np.array_equal(x[idx].view(np.uint8), vals.view(np.uint8))
    mask = np.ones(x.size, bool)
    mask[idx] = False
    if mask.any():
        if select_min:
            assert vals.max() <= x[mask].min()
        else:
            assert vals.min() >= x[mask].max()


# ---------------------------------------------------------------------------------------------
# order-preserving code: pinned by exhaustive enumeration against the hardware float order

def test_code_f16_exhaustive_matches_float_order():
    bits = f16_all()
    c = oracle.codes(bits, dt=oracle.DT_NAMES["f16"]).astype(np.int64)
    assert np.array_equal(np.sort(c), np.arange(1 << 16))            # bijection on 16 bits
    order = np.argsort(c)
    v = bits[order].view(np.float16).astype(np.float64)
    finite = ~np.isnan(v)
    vv = v[finite]
    assert np.all(np.diff(vv) >= 0)                                   # monotone in IEEE order
    # the only equal neighbours are -0, +0 and -0 comes first
    eq = np.flatnonzero(np.diff(vv) == 0)
    assert eq.size == 1
    b_ord = bits[order][finite]
    assert b_ord[eq[0]] == 0x8000 and b_ord[eq[0] + 1] == 0x0000
    # NaNs: negative-signed below -inf, positive-signed above +inf
    nan_pos = np.flatnonzero(~finite)
    sign = (bits[order][~finite] >> 15) & 1
    assert np.all(nan_pos[sign == 1] < np.flatnonzero(v == -np.inf)[0])
    assert np.all(nan_pos[sign == 0] > np.flatnonzero(v == np.inf)[0])


def test_code_bf16_exhaustive_matches_float_order():
    bits = f16_all()
    c = oracle.codes(bits, dt=oracle.DT_NAMES["bf16"]).astype(np.int64)
    assert np.array_equal(np.sort(c), np.arange(1 << 16))
    order = np.argsort(c)
    v = (bits[order].astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    vv = v[~np.isnan(v)]
    assert np.all(np.diff(vv) >= 0)
    assert np.count_nonzero(np.diff(vv) == 0) == 1


def test_code_select_max_reverses_order():
    x = gen.normal_f32(7, 4096)
    cmin = oracle.codes(x, select_min=True)
    cmax = oracle.codes(x, select_min=False)
    assert np.array_equal(np.argsort(cmin.reshape(-1), kind="stable"), np.argsort(x, kind="stable"))
    assert np.all((cmin.astype(np.uint64) ^ cmax.astype(np.uint64)) == np.uint64(0xFFFFFFFF))


def test_code_u32_identity():
    u = gen.u32(3, 1000)
    assert np.array_equal(oracle.codes(u).astype(np.uint32), u)


# ---------------------------------------------------------------------------------------------
# selected set: pinned by numpy's stable argsort (ties -> lowest index) on NaN-free inputs

@pytest.mark.parametrize("dist", ["uniform", "normal", "adversarial"])
@pytest.mark.parametrize("k", [1, 17, 1000])
@pytest.mark.parametrize("select_min", [True, False])
def test_sort_oracle_equals_numpy_stable_argsort(dist, k, select_min):
    x = gen.keys(dist, 11, 1 << 14)
    x = np.where(x == 0, np.float32(1e-30), x)        # avoid -0/+0, which numpy treats as equal
    key = x.astype(np.float64) if select_min else -x.astype(np.float64)
    ref = np.argsort(key, kind="stable")[:k]
    vals, idx = oracle.topk_sort(x, k, select_min)
    assert np.array_equal(idx[0], ref)
    assert np.array_equal(vals[0], x[ref])
    check_definition_f(x, vals[0], idx[0], k, select_min)


def test_f64_and_u32_equal_numpy():
    x = gen.uniform_f64(5, 5000)
    _, idx = oracle.topk_nth(x, 123)
    assert np.array_equal(idx[0], np.argsort(x, kind="stable")[:123])
    u = gen.u32(5, 5000) % 97        # many ties
    _, idx = oracle.topk_nth(u, 300, select_min=False)
    assert np.array_equal(idx[0], np.argsort(-u.astype(np.int64), kind="stable")[:300])


# three independent derivations (sort / nth_element / O(N^2) rank) on adversarial bit patterns

_dt_pool = st.sampled_from(["f32", "f16", "bf16", "f64", "u32"])


def _raw(dtn, seed, n, pool):
    w = {"f32": 4, "f16": 2, "bf16": 2, "f64": 8, "u32": 4}[dtn]
    bits = gen.u64(seed, n)
    if pool:
        bits = gen.u64(seed + 1, pool)[bits % np.uint64(pool)]   # heavy ties
    arr = bits.astype({2: np.uint16, 4: np.uint32, 8: np.uint64}[w])
    return arr


@settings(max_examples=60, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(dtn=_dt_pool, n=st.integers(1, 300), kfrac=st.floats(0, 1), seed=st.integers(0, 1 << 30),
       pool=st.sampled_from([0, 1, 2, 7]), select_min=st.booleans(), batch=st.integers(1, 3))
def test_three_oracles_agree(dtn, n, kfrac, seed, pool, select_min, batch):
    k = max(1, min(n, int(round(kfrac * n))))
    raw = _raw(dtn, seed, n * batch, pool).reshape(batch, n)
    dt = oracle.DT_NAMES[dtn]
    a = oracle.topk_sort(raw, k, select_min, dt=dt)
    b = oracle.topk_nth(raw, k, select_min, dt=dt)
    c = oracle.topk_brute(raw, k, select_min, dt=dt)
    d = oracle.topk_nth_mt(raw, k, select_min, dt=dt)[:2]
    for x, y in ((a, b), (a, c), (a, d)):
        assert np.array_equal(x[0], y[0]) and np.array_equal(x[1], y[1])


def test_nth_mt_matches_sort_on_large_tied_rows():
    """The all-cores baseline variant (chunked nth_element + merge) equals the sort oracle where
    chunks cut through long runs of ties (a wrong chunk merge or tie rule would differ)."""
    x = gen.adversarial_f32(5, 300_001, m_bits=26)      # 64 distinct values, ~4.7K ties each
    for k in (1, 999, 4688, 50_000, 300_001):
        a = oracle.topk_sort(x, k)
        v, i, th = oracle.topk_nth_mt(x, k)
        assert th >= 1
        assert np.array_equal(a[0], v) and np.array_equal(a[1], i)


# ---------------------------------------------------------------------------------------------
# closed forms on tie-heavy inputs (PAPER.md:162-164 radix-adversarial; PAPER.md:186 K == N)

def test_adversarial_closed_form():
    # M = 24: 256 distinct values, each ~4096 times in 2^20; K below the count of the minimum
    x = gen.adversarial_f32(20231116, 1 << 20, m_bits=24)
    assert np.all((x.view(np.uint32) >> 8) == (0x3F800000 >> 8))
    k = 1000
    vals, idx = oracle.topk_nth(x, k)
    first = np.flatnonzero(x == np.float32(1.0))
    assert first.size > k
    assert np.all(vals[0].view(np.uint32) == 0x3F800000)
    assert np.array_equal(idx[0], first[:k])


def test_all_equal_and_k_equals_n():
    x = np.full(1000, 3.5, np.float32)
    _, idx = oracle.topk_nth(x, 10)
    assert np.array_equal(idx[0], np.arange(10))
    y = gen.normal_f32(1, 777)
    vals, idx = oracle.topk_nth(y, 777)
    assert np.array_equal(np.sort(idx[0]), np.arange(777))


def test_invalid_args_rejected():
    x = np.zeros(10, np.float32)
    for k in (0, 11):
        with pytest.raises(ValueError):
            oracle.topk_sort(x, k)


# ---------------------------------------------------------------------------------------------
# with_idx (multi-GPU merge): merge of per-shard top-K == single-row top-K (SURVEY §8(e) argument)

@pytest.mark.parametrize("shards", [2, 3, 8])
@pytest.mark.parametrize("dist", ["uniform", "adversarial"])
def test_shard_merge_equals_single_row(shards, dist):
    n, k = 6000, 500
    x = gen.keys(dist, 99, n, m_bits=28)
    bounds = np.linspace(0, n, shards + 1).astype(int)
    cv, ci = [], []
    for s in range(shards):
        lo, hi = bounds[s], bounds[s + 1]
        kk = min(k, hi - lo)
        v, i = oracle.topk_sort(x[lo:hi], kk)
        cv.append(v[0]); ci.append(i[0] + lo)
    # gather in reverse shard order so position order != global index order
    gv = np.concatenate(cv[::-1]); gi = np.concatenate(ci[::-1])
    mv, mi = oracle.topk_with_idx(gv, gi, k)
    rv, ri = oracle.topk_sort(x, k)
    assert np.array_equal(mi, ri[0]) and np.array_equal(mv.view(np.uint32), rv[0].view(np.uint32))


# ---------------------------------------------------------------------------------------------
# Algorithm 1 trace

def test_fig1_worked_example():
    g = json.load(open(os.path.join(GOLD, "fig1_radix_example.json")))
    codes = np.array(g["codes"], np.uint64)
    sel, recs, hists = oracle.radix_trace(codes, g["k"], r_bits=g["r_bits"], b=g["b"], alpha=1 << 30)
    r1, r2 = recs[0], recs[1]
    assert list(hists[0][:4]) == g["iter1"]["hist"]
    assert list(np.cumsum(hists[0][:4])) == g["iter1"]["psum"]
    assert r1["j"] == g["iter1"]["target_digit"] and r1["K"] == g["iter1"]["K_after"] and r1["C"] == g["iter1"]["C_after"]
    assert list(hists[1][:4]) == g["iter2"]["hist"]
    assert r2["j"] == g["iter2"]["target_digit"] and r2["K"] == 1 and r2["C"] == 1 and r2["early_stop"] == 1
    assert r2["emitted"] == 2          # the two '00' elements are emitted by the iteration-2 filter
    assert list(codes[sel]) == g["selected_codes_sorted"]
    assert list(sel) == g["selected_idx_sorted_by_code"]


def _bincount_prefix(c, shift, width, pshift=None, prefix=None):
    d = (c >> np.uint64(shift)) & np.uint64((1 << width) - 1)
    if pshift is not None:
        d = d[(c >> np.uint64(pshift)) == np.uint64(prefix)]
    return np.bincount(d.astype(np.int64), minlength=1 << 11)


@pytest.mark.parametrize("dist", ["uniform", "normal", "adversarial"])
def test_trace_histograms_match_brute_force(dist):
    """Per-pass histogram = brute-force count of the digit over the elements whose higher digits
    equal the chosen targets."""
    x = gen.keys(dist, 5, 1 << 18)
    c = oracle.codes(x)[0] if x.ndim > 1 else oracle.codes(x)
    c = c.reshape(-1)
    k = 333
    sel, recs, hists = oracle.radix_trace(c, k, early_stop=False)
    j1, j2 = recs[0]["j"], recs[1]["j"]
    assert np.array_equal(hists[0], _bincount_prefix(c, 21, 11))
    assert np.array_equal(hists[1], _bincount_prefix(c, 10, 11, 21, j1))
    assert np.array_equal(hists[2], _bincount_prefix(c, 0, 10, 10, (j1 << 11) | j2))
    # invariants: C >= K >= 1; final prefix is the K-th smallest code
    for r in recs[:-1]:
        assert r["C"] >= r["K"] >= 1
    kth = np.sort(c)[k - 1]
    assert (recs[0]["j"] << 21) | (recs[1]["j"] << 10) | recs[2]["j"] == int(kth)
    assert recs[2]["K"] == k - int(np.count_nonzero(c < kth))


@pytest.mark.parametrize("dist,m", [("uniform", 0), ("normal", 0), ("adversarial", 20), ("adversarial", 10)])
@pytest.mark.parametrize("alpha", [1, 4, 128, 1 << 40])
@pytest.mark.parametrize("early", [True, False])
@pytest.mark.parametrize("idx_bits", [0, 16])
def test_trace_reaches_definition(dist, m, alpha, early, idx_bits):
    """Algorithm 1 + adaptive buffering + early stop selects exactly the definition's set, for any
    alpha (result independent of buffering) and with early stop on or off
    (PAPER.md:186), and with ties resolved by extra index digits or by the last filter."""
    n = 1 << 16
    x = gen.keys(dist, 17, n, m_bits=m or 20)
    c = oracle.codes(x).reshape(-1)
    for k in (1, 32, 5000, n):
        sel, recs, _ = oracle.radix_trace(c, k, idx_bits=idx_bits, alpha=alpha, early_stop=early)
        _, ref = oracle.topk_sort(x, k)
        assert np.array_equal(sel, ref[0])
        for r in recs[:-1]:
            # buffer never holds more than N/alpha
            if r["stored"]:
                assert r["Cp"] * alpha < n


def test_trace_adaptive_worst_case_reads():
    """Radix-adversarial M=20: no candidate is eliminated by pass 1, so every
    kernel re-reads L: 2G_1 + sum G_i with G_i = N, and nothing is ever buffered
    while C >= N/alpha."""
    n = 1 << 20
    x = gen.adversarial_f32(20231116, n, m_bits=20)
    c = oracle.codes(x).reshape(-1)
    k = 50
    sel, recs, _ = oracle.radix_trace(c, k, alpha=128)
    assert recs[0]["C"] == n                  # first 11 bits identical
    assert [r["read"] for r in recs[:3]] == [n, n, n]
    assert recs[0]["src_L"] and recs[1]["src_L"] and not recs[1]["stored"]
    # uniform: pass 2 buffers (C1 << N/alpha), pass 3 reads the buffer
    u = gen.uniform_f32(20231113, n)
    cu = oracle.codes(u).reshape(-1)
    _, ru, _ = oracle.radix_trace(cu, 1 << 10, alpha=128, early_stop=False)
    assert ru[1]["stored"] == 1 and ru[2]["src_L"] == 0 and ru[2]["read"] == ru[0]["C"]


def test_trace_never_buffer_when_alpha_is_n():
    """alpha = N ensures no candidate buffer is required."""
    n = 1 << 14
    x = gen.uniform_f32(3, n)
    c = oracle.codes(x).reshape(-1)
    _, recs, _ = oracle.radix_trace(c, 100, alpha=n)
    assert all(r["stored"] == 0 for r in recs) and all(r["src_L"] == 1 for r in recs)


def test_trace_early_stop_when_k_equals_c():
    x = np.array([5, 1, 1, 1, 9, 9], np.uint32)       # K = 4: ties fill K exactly after pass 3
    c = oracle.codes(x).reshape(-1)
    sel, recs, _ = oracle.radix_trace(c, 4)
    stops = [r["early_stop"] for r in recs[:-1]]
    assert stops[-1] == 1 and recs[len(stops) - 1]["K"] == recs[len(stops) - 1]["C"]
    assert sorted(sel.tolist()) == [0, 1, 2, 3]
