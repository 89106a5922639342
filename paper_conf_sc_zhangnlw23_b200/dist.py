"""Multi-GPU AIR Top-K over torch.distributed (one process per GPU, NCCL over NVLink/NVSwitch).

Only the two natural partitionings exist:

* select_rows — a batch of independent rows is split into contiguous row blocks, one per
  rank; every rank selects its own rows. No data-path collective at all.
* select_split_row — one huge row is split into contiguous shards; every rank selects the local
  top-K of its shard (row-local ties -> lowest local index == lowest global index inside the
  shard), the K candidates of every rank are all-gathered as packed (value bits, global index)
  pairs (the ONE exchange step: one NCCL all_gather over NVLink), and a merge select over the
  world*K candidates, ties ranked by the global index value, gives the global top-K on every rank. Exact: a global top-K element has
  fewer than K predecessors in (code, global index) order, hence fewer than K in its own shard,
  so it is in that shard's local top-K.

`select_fn` / `merge_fn` are injectable so the partition/gather/merge logic can be tested on CPU
with the gloo backend; the product path uses the CUDA kernels of libairtopk.so.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import select, select_with_idx


def row_range(batch: int, rank: int, world: int):
    """Contiguous row block [lo, hi) of `rank` (rows differ by at most one between ranks)."""
    return batch * rank // world, batch * (rank + 1) // world


def select_rows(x_local, k: int, largest: bool = False, group=None, select_fn=None, **kw):
    """Top-K of every local row; returns (values, row-local indices, first global row)."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    fn = select_fn or (lambda t, kk, lg: select(t, kk, largest=lg, **kw))
    v, i = fn(x_local, k, largest)
    return v, i, rank  # caller knows its row offset from row_range; rank returned for convenience


def pad_bits(dtype, largest: bool) -> int:
    """Bit pattern of the element that sorts LAST in the selection order (max code): +NaN with a
    full payload for select-min, -NaN with a full payload for select-max (u32: max / 0)."""
    r = {torch.float32: 32, torch.float16: 16, torch.bfloat16: 16, torch.float64: 64, torch.uint32: 32}[dtype]
    if dtype == torch.uint32:
        return 0 if largest else 0xFFFFFFFF
    full = (1 << r) - 1
    return full if largest else full >> 1


def _bits_view(t):
    m = {1: torch.uint8, 2: torch.int16, 4: torch.int32, 8: torch.int64}
    return t.view(m[t.element_size()])


def _all_gather(t, group):
    world = dist.get_world_size(group)
    if dist.get_backend(group) == "nccl":
        out = torch.empty((world,) + tuple(t.shape), dtype=t.dtype, device=t.device)
        dist.all_gather_into_tensor(out, t.contiguous(), group=group)
        return out
    # gloo (CPU tests, or the multi-rank self-test of bench.py): gather through host memory
    tc = t.contiguous().cpu()
    parts = [torch.empty_like(tc) for _ in range(world)]
    dist.all_gather(parts, tc, group=group)
    return torch.stack(parts).to(t.device)


def select_split_row(x_shard, k: int, total_len: int, shard_offset: int, largest: bool = False, group=None,
                     select_fn=None, merge_fn=None):
    """Global top-K of a row split across ranks. x_shard: this rank's contiguous shard (1-D),
    starting at global index shard_offset; total_len: length of the whole row.
    Returns (values [k], global indices [k]) on every rank."""
    x_shard = x_shard.reshape(-1)
    n = x_shard.numel()
    kk = min(k, n)
    fn = select_fn or (lambda t, kq, lg: select(t, kq, largest=lg))
    v, i = fn(x_shard, kk, largest)
    v = v.reshape(-1)
    gidx = i.reshape(-1).to(torch.int64) + shard_offset
    if kk < k:  # pad so every rank contributes exactly k candidates (they sort last, never selected)
        pad = k - kk
        bits = pad_bits(x_shard.dtype, largest)
        width = 8 * v.element_size()
        if bits >= 1 << (width - 1):  # as the signed integer of the same width
            bits -= 1 << width
        pv = torch.full((pad,), bits, dtype=_bits_view(v).dtype, device=v.device)
        v = torch.cat([v, pv.view(v.dtype)])
        rank = dist.get_rank(group)
        gidx = torch.cat([gidx, total_len + rank * k + torch.arange(pad, dtype=torch.int64, device=gidx.device)])
    world = dist.get_world_size(group)
    # ONE all-gather of packed (value bits, global index) pairs: [k, 2] int64 per rank
    vb = _bits_view(v)
    packed = torch.stack([vb.to(torch.int64), gidx], dim=1)
    g = _all_gather(packed, group).reshape(-1, 2)
    gv = g[:, 0].to(vb.dtype).view(v.dtype)
    gi = g[:, 1].contiguous()
    idx_bits = max(1, int(total_len + world * k - 1).bit_length())
    mfn = merge_fn or (lambda a, b, kq, ib, lg: select_with_idx(a, b, kq, ib, largest=lg))
    return mfn(gv, gi, k, idx_bits, largest)
