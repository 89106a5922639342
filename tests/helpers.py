"""Shared test helpers: move seeded inputs to the GPU, call the CUDA path through the C ABI
binding, and compare with the CPU oracle bit-exactly (identical value multiset, identical index
set under the lowest-index tie rule)."""
from __future__ import annotations

import numpy as np

import oracle

BITS_NP = {"f32": np.uint32, "f16": np.uint16, "bf16": np.uint16, "f64": np.uint64, "u32": np.uint32}


def torch_dtype(dtn):
    import torch
    return {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16, "f64": torch.float64,
            "u32": torch.uint32}[dtn]


def to_device(raw_bits: np.ndarray, dtn: str, offset_elems: int = 0):
    """Device tensor with the given raw bit patterns. offset_elems > 0 returns a view starting
    that many elements into a larger allocation (misaligned data pointer)."""
    import torch
    raw = np.ascontiguousarray(raw_bits).view(BITS_NP[dtn])
    signed = {np.uint16: np.int16, np.uint32: np.int32, np.uint64: np.int64}[BITS_NP[dtn]]
    flat = raw.reshape(-1).view(signed)
    if offset_elems:
        flat = np.concatenate([np.zeros(offset_elems, signed), flat])
    t = torch.from_numpy(flat.copy()).cuda().view(torch_dtype(dtn))
    t = t[offset_elems:]
    return t.reshape(raw.shape)


def to_bits(t, dtn) -> np.ndarray:
    import torch
    signed = {"f32": torch.int32, "f16": torch.int16, "bf16": torch.int16, "f64": torch.int64, "u32": torch.int32}[dtn]
    return t.contiguous().view(signed).cpu().numpy().view(BITS_NP[dtn])


def gpu_select(raw_bits, dtn, k, select_min=True, offset_elems=0, **kw):
    import paper_conf_sc_zhangnlw23_b200 as at
    x = to_device(raw_bits, dtn, offset_elems)
    if x.dim() == 1:
        x = x.reshape(1, -1)
    v, i = at.select(x, k, largest=not select_min, **kw)
    import torch
    torch.cuda.synchronize()
    return to_bits(v, dtn), i.cpu().numpy()


def assert_parity(raw_bits, dtn, k, select_min, gvals, gidx, ref=None):
    raw = np.ascontiguousarray(raw_bits).view(BITS_NP[dtn])
    if raw.ndim == 1:
        raw = raw[None, :]
    batch, n = raw.shape
    gvals = gvals.reshape(batch, k)
    gidx = gidx.reshape(batch, k)
    if ref is None:
        ref = oracle.topk_nth(raw, k, select_min, dt=oracle.DT_NAMES[dtn])
    rv, ri = ref
    for r in range(batch):
        order = np.argsort(gidx[r], kind="stable")
        gi = gidx[r][order]
        assert gi.min() >= 0 and gi.max() < n, f"row {r}: index out of range"
        assert np.array_equal(gvals[r][order], raw[r][gi]), f"row {r}: value bits do not match keys[idx]"
        ro = np.argsort(ri[r], kind="stable")
        if not np.array_equal(gi, ri[r][ro]):
            bad = np.setdiff1d(gi, ri[r])
            raise AssertionError(f"row {r}: index sets differ ({bad.size} extra, e.g. {bad[:5]})")
        assert np.array_equal(np.sort(gvals[r]), np.sort(rv[r].view(BITS_NP[dtn])))
