"""Multi-GPU AIR Top-K over torch.distributed (one process per GPU, NCCL over NVLink/NVSwitch).

Only the two natural partitionings exist:

* select_rows — a batch of independent rows is split into contiguous row blocks, one per
  rank; every rank selects its own rows. No data-path collective at all.
* select_split_row — one huge row is split into contiguous shards (the top 0.1 % of a
  gradient spread over workers). Every rank runs airtopk_select_shard on its shard: the kernels
  write the shard's k best keys with GLOBAL indices (local + shard offset; ties -> lowest index)
  straight into this rank's slot of the gather buffers, plus pad entries that sort last when the
  shard is shorter than k. ONE coalesced NCCL all-gather (values + indices, in place) is the only
  exchange step; airtopk_select_with_idx over the world*k gathered candidates, ties ranked by the
  global index value, then gives the global top-k on every rank. Exact: a global top-k element has
  fewer than k predecessors in (code, global index) order, hence fewer than k in its own shard, so
  it is in that shard's local top-k.

Torch provides only device memory, streams and the process group: every arithmetic step (local
select, index offset, padding, merge) runs in libairtopk.so kernels. `shard_fn` / `merge_fn` are
injectable so the gather / merge flow can be tested on CPU with the gloo backend.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import merge_idx_bits, select, select_shard, select_with_idx


def row_range(batch: int, rank: int, world: int):
    """Contiguous row block [lo, hi) of `rank` (rows differ by at most one between ranks)."""
    return batch * rank // world, batch * (rank + 1) // world


def select_rows(x_local, k: int, largest: bool = False, group=None, select_fn=None, **kw):
    """Top-K of every local row; returns (values, row-local indices, rank)."""
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    fn = select_fn or (lambda t, kk, lg: select(t, kk, largest=lg, **kw))
    v, i = fn(x_local, k, largest)
    return v, i, rank  # the caller knows its row offset from row_range


def pad_bits(dtype, largest: bool) -> int:
    """Bit pattern of the element that sorts LAST in the selection order (max code): +NaN with a
    full payload for select-min, -NaN with a full payload for select-max (u32: max / 0). The
    kernels write the same pattern (airtopk_select_shard); this is the host-side statement of it."""
    r = {torch.float32: 32, torch.float16: 16, torch.bfloat16: 16, torch.float64: 64, torch.uint32: 32}[dtype]
    if dtype == torch.uint32:
        return 0 if largest else 0xFFFFFFFF
    full = (1 << r) - 1
    return full if largest else full >> 1


def all_gather_inplace(tensors, group=None):
    """In-place all-gather of several [world * n] buffers whose slot `rank` holds this rank's part:
    one NCCL group (coalesced) on NCCL; per-buffer all_gather through host memory on gloo."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if dist.get_backend(group) == "nccl":
        from torch.distributed.distributed_c10d import _coalescing_manager
        with _coalescing_manager(group, tensors[0].device):
            for t in tensors:
                n = t.numel() // world
                dist.all_gather_into_tensor(t, t[rank * n:(rank + 1) * n], group=group)
        return
    for t in tensors:  # gloo (CPU tests, or the multi-rank self-test of bench.py on one GPU)
        n = t.numel() // world
        parts = [torch.empty(n, dtype=t.dtype) for _ in range(world)]
        dist.all_gather(parts, t[rank * n:(rank + 1) * n].cpu(), group=group)
        t.copy_(torch.cat(parts).to(t.device))


def select_split_row(x_shard, k: int, total_len: int, shard_offset: int, largest: bool = False, group=None,
                     shard_fn=None, merge_fn=None, buffers=None):
    """Global top-K of a row split across ranks. x_shard: this rank's contiguous shard (1-D),
    starting at global index shard_offset; total_len: length of the whole row.
    Returns (values [k], global indices [k]) on every rank. `buffers` = (vals [world*k],
    idx [world*k] int64) gather buffers to reuse (allocated if None)."""
    x_shard = x_shard.reshape(-1)
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if buffers is None:
        buffers = (torch.empty(world * k, dtype=x_shard.dtype, device=x_shard.device),
                   torch.empty(world * k, dtype=torch.int64, device=x_shard.device))
    gv, gi = buffers
    mine = slice(rank * k, (rank + 1) * k)
    pad_base = total_len + rank * k  # pad indices never collide across ranks
    fn = shard_fn or (lambda t, kk, off, pb, lg, out: select_shard(t, kk, off, pb, largest=lg, out=out))
    fn(x_shard, k, shard_offset, pad_base, largest, (gv[mine], gi[mine]))
    all_gather_inplace([gv, gi], group)
    idx_bits = merge_idx_bits(total_len, world, k)
    mfn = merge_fn or (lambda a, b, kq, ib, lg: select_with_idx(a, b, kq, ib, largest=lg))
    return mfn(gv, gi, k, idx_bits, largest)


class PeerExchange:
    """Collective-fused split-row exchange: gather buffers [world * k] and a
    flag array on every rank, opened by every peer through CUDA IPC (handles exchanged once with
    all_gather_object over `group`). exchange() = ONE push kernel (this rank's k entries stored into
    slot `rank` of every rank's buffers, then its flag raised in every rank) + ONE wait kernel (all
    flags carry this call's epoch) — no NCCL collective. Every rank must call exchange() in the same
    order (the epoch is a call counter)."""

    def __init__(self, k: int, dtype, device, group=None):
        import ctypes
        from . import dtype_code, lib
        self.lib = lib()
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.k = k
        self.dt = dtype_code(dtype)
        self.vals = torch.empty(self.world * k, dtype=dtype, device=device)
        self.idx = torch.empty(self.world * k, dtype=torch.int64, device=device)
        self.flags = torch.zeros(self.world, dtype=torch.int32, device=device)
        self.ticket = torch.zeros(1, dtype=torch.int32, device=device)
        torch.cuda.synchronize(device)
        mine = []
        for t in (self.vals, self.idx, self.flags):
            h = (ctypes.c_char * 64)()
            off = ctypes.c_uint64(0)
            st = self.lib.airtopk_ipc_handle(t.data_ptr(), h, ctypes.byref(off))
            if st != 0:
                raise RuntimeError(f"airtopk_ipc_handle failed ({st})")
            mine.append((bytes(h), int(off.value)))
        allh = [None] * self.world
        dist.all_gather_object(allh, mine, group=group)
        self.opened = []
        ptrs = [[], [], []]
        for r in range(self.world):
            for b, t in enumerate((self.vals, self.idx, self.flags)):
                if r == self.rank:
                    ptrs[b].append(t.data_ptr())
                    continue
                hb, off = allh[r][b]
                p = ctypes.c_void_p()
                st = self.lib.airtopk_ipc_open((ctypes.c_char * 64).from_buffer_copy(hb), off, ctypes.byref(p))
                if st != 0:
                    raise RuntimeError(f"airtopk_ipc_open failed ({st})")
                self.opened.append(p.value)
                ptrs[b].append(p.value)
        arr = lambda xs: (ctypes.c_void_p * self.world)(*xs)
        self.peer_vals, self.peer_idx, self.peer_flags = arr(ptrs[0]), arr(ptrs[1]), arr(ptrs[2])
        self.epoch = 0
        dist.barrier(group=group)

    def slot(self):
        """(values, indices) views of this rank's slot: the shard select writes here."""
        s = slice(self.rank * self.k, (self.rank + 1) * self.k)
        return self.vals[s], self.idx[s]

    def exchange(self, stream=None):
        self.epoch = (self.epoch + 1) & 0xFFFFFFFF or 1
        s = (stream if stream is not None else torch.cuda.current_stream(self.vals.device)).cuda_stream
        v, i = self.slot()
        st = self.lib.airtopk_shard_push(v.data_ptr(), i.data_ptr(), self.k, self.dt, self.world, self.rank,
                                         self.peer_vals, self.peer_idx, self.peer_flags, self.epoch,
                                         self.ticket.data_ptr(), s)
        if st != 0:
            raise RuntimeError(f"airtopk_shard_push failed ({st})")
        st = self.lib.airtopk_wait_flags(self.flags.data_ptr(), self.world, self.epoch, s)
        if st != 0:
            raise RuntimeError(f"airtopk_wait_flags failed ({st})")

    def close(self):
        for p in self.opened:
            self.lib.airtopk_ipc_close(p)
        self.opened = []


def select_split_row_p2p(x_shard, k: int, total_len: int, shard_offset: int, ex: PeerExchange, largest: bool = False,
                         workspace=None, merge_workspace=None, out=None):
    """select_split_row with the exchange over peer memory (PeerExchange) instead of NCCL."""
    x_shard = x_shard.reshape(-1)
    pad_base = total_len + ex.rank * k
    select_shard(x_shard, k, shard_offset, pad_base, largest=largest, out=ex.slot(), workspace=workspace)
    ex.exchange()
    return select_with_idx(ex.vals, ex.idx, k, merge_idx_bits(total_len, ex.world, k), largest=largest,
                           workspace=merge_workspace, out=out)
