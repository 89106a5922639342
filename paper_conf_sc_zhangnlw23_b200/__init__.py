"""B200-native AIR Top-K (Zhang et al., SC'23) — thin Python binding over libairtopk.so.

Every step of the selection runs in the CUDA kernels of libairtopk.so (csrc/); this module only
marshals torch tensors (device memory, the current stream) into the C ABI of include/airtopk.h.
There is no CPU fallback: calling without the built library or on a CPU tensor raises.

    values, indices = select(x, k, largest=False)      # x: [batch, len] or [len] CUDA tensor
"""
from __future__ import annotations

import contextlib
import ctypes

from . import _lib
from ._lib import (AirTopKError, Options, OK, ENGINE_AUTO, ENGINE_GRID, ENGINE_CLUSTER, ENGINE_GRIDSELECT,
                   ENGINE_BATCH, ENGINE_RESIDENT, ENGINE_GRIDSELECT_PTQ, TRACE_MAX_PASSES)

__all__ = ["select", "select_with_idx", "select_shard", "merge_idx_bits", "select_host", "workspace_bytes",
           "describe", "lib", "AirTopKError", "DeviceError", "ENGINE_AUTO", "ENGINE_GRID", "ENGINE_CLUSTER",
           "ENGINE_GRIDSELECT", "ENGINE_BATCH", "ENGINE_RESIDENT", "ENGINE_GRIDSELECT_PTQ", "dtype_code"]

_LIB = None


class DeviceError(RuntimeError):
    """The kernels flagged an inconsistency (AIRTOPK_ERR_* bits), e.g. duplicate in_idx values."""

    def __init__(self, bits: int):
        names = [n for b, n in ((_lib.ERR_OUTPUT_OVERFLOW, "more than K results"),
                                (_lib.ERR_BUFFER_OVERFLOW, "candidate buffer overflow"),
                                (_lib.ERR_COUNT, "count mismatch / fewer than K results")) if bits & b]
        super().__init__(f"AIR Top-K device status 0x{bits:x}: " + ", ".join(names))
        self.bits = bits


def lib():
    """The loaded libairtopk.so (raises ImportError if it was not built)."""
    global _LIB
    if _LIB is None:
        _LIB = _lib.load()
    return _LIB


def _torch():
    import torch
    return torch


_DTYPES = None
_NULLCTX = contextlib.nullcontext()


def dtype_code(dtype) -> int:
    global _DTYPES
    if _DTYPES is None:
        torch = _torch()
        _DTYPES = {torch.float32: _lib.F32, torch.float16: _lib.F16, torch.bfloat16: _lib.BF16,
                   torch.float64: _lib.F64, torch.uint32: _lib.U32}
    c = _DTYPES.get(dtype)
    if c is None:
        raise TypeError(f"unsupported key dtype {dtype} (f32/f16/bf16/f64/u32)")
    return c


def _check(status: int):
    if status != OK:
        if status in (_lib.EINVAL, _lib.EDTYPE, _lib.ENOSPACE):
            raise _lib.AirTopKArgumentError(status, lib())
        raise AirTopKError(status, lib())


_OPTS_CACHE = {}


def _opts(alpha=0, engine=ENGINE_AUTO, ctas_per_row=0, cluster_size=0, trace=None, events=None, window=0, tma=0,
          early_stop=0, status=None, sorted_out=False):
    if trace is None and events is None and status is None:
        # pointer-free options are immutable once built: one ctypes struct per distinct tuple (the
        # per-call cost of the binding matters for latency-bound rows: c1 is ~12 us on the GPU)
        key = (alpha, engine, ctas_per_row, cluster_size, window, tma, early_stop, sorted_out)
        o = _OPTS_CACHE.get(key)
        if o is None:
            o = _OPTS_CACHE[key] = _build_opts(*key)
        return o
    o = _build_opts(alpha, engine, ctas_per_row, cluster_size, window, tma, early_stop, sorted_out)
    o.trace = trace.data_ptr() if trace is not None else None
    o.trace_len = trace.numel() if trace is not None else 0
    o.status = status.data_ptr() if status is not None else None
    if events is not None:
        # events: a ctypes array of cudaEvent_t handles (see make_event_array)
        o.events = ctypes.cast(events, ctypes.c_void_p)
        o.n_events = len(events)
    return o


def _build_opts(alpha, engine, ctas_per_row, cluster_size, window, tma, early_stop, sorted_out):
    o = Options()
    o.sorted = 1 if sorted_out else 0
    o.early_stop = int(early_stop)
    o.window = int(window)
    o.tma = int(tma)
    o.alpha = int(alpha)
    o.engine = int(engine)
    o.ctas_per_row = int(ctas_per_row)
    o.cluster_size = int(cluster_size)
    return o


def make_event_array(events):
    """ctypes array of the raw cudaEvent_t handles of torch.cuda.Event objects (already created)."""
    arr = (ctypes.c_void_p * len(events))()
    for j, e in enumerate(events):
        arr[j] = e.cuda_event
    return arr


def workspace_bytes(dtype, batch: int, length: int, k: int, alpha: int = 0, **kw) -> int:
    o = _opts(alpha, **kw)
    return int(lib().airtopk_workspace_bytes_ex(dtype_code(dtype), batch, length, k, ctypes.byref(o)))


def describe(dtype, batch: int, length: int, k: int, alpha: int = 0, engine: int = ENGINE_AUTO,
             ctas_per_row: int = 0, cluster_size: int = 0, window: int = 0, tma: int = 0, early_stop: int = 0) -> dict:
    """How a select with these arguments runs: engine, passes, launches, grid shape, workspace."""
    o = _opts(alpha, engine, ctas_per_row, cluster_size, window=window, tma=tma, early_stop=early_stop)
    pl = _lib.Plan()
    _check(lib().airtopk_describe(dtype_code(dtype), batch, length, k, ctypes.byref(o), ctypes.byref(pl)))
    return {f: getattr(pl, f) for f, _ in _lib.Plan._fields_}


def _stream(stream, device):
    torch = _torch()
    if stream is None:  # the raw cudaStream_t of torch's current stream (no Stream object built)
        raw = getattr(torch._C, "_cuda_getCurrentRawStream", None)
        return raw(device.index) if raw is not None else torch.cuda.current_stream(device).cuda_stream
    if stream.device != device:
        raise ValueError(f"stream of {stream.device} used with tensors on {device}")
    return stream.cuda_stream


def _check_out(t, shape, dtype, device, what):
    if t.shape != shape or t.dtype != dtype or t.device != device or not t.is_contiguous():
        raise ValueError(f"{what} must be a contiguous {dtype} tensor of shape {tuple(shape)} on {device} "
                         f"(got {t.dtype} {tuple(t.shape)} on {t.device}, contiguous={t.is_contiguous()})")


def _workspace(workspace, need, device):
    torch = _torch()
    if workspace is None:
        return torch.empty(max(need, 1), dtype=torch.uint8, device=device) if need else None
    if workspace.dtype != torch.uint8 or workspace.device != device or not workspace.is_contiguous():
        raise ValueError(f"workspace must be a contiguous uint8 tensor on {device}")
    if workspace.numel() < need:
        raise ValueError(f"workspace has {workspace.numel()} bytes, {need} needed")
    return workspace


def _status_word(check, status, device):
    torch = _torch()
    if status is not None:
        if status.dtype not in (torch.int32, torch.uint32) or status.device != device or status.numel() != 1:
            raise ValueError("status must be a 1-element int32/uint32 tensor on the keys' device")
        return status
    if check:
        return torch.zeros(1, dtype=torch.int32, device=device)
    return None


def _raise_status(st):
    bits = int(st.view(_torch().int32).item()) & 0xFFFFFFFF
    if bits:
        raise DeviceError(bits)


def select(x, k: int, largest: bool = False, *, alpha: int = 0, engine: int = ENGINE_AUTO,
           ctas_per_row: int = 0, cluster_size: int = 0, trace=None, events=None, window: int = 0,
           tma: int = 0, early_stop: int = 0, workspace=None, out=None, stream=None, status=None,
           check: bool = False, sorted: bool = False):
    """Top-K of each row of `x` ([batch, len] or [len], contiguous CUDA tensor).

    Returns (values, indices): [batch, k] of x.dtype (raw bit copies) and int64 row-local indices,
    order within a row unspecified. Ties at the K-th value go to the lowest index. Enqueued on
    `stream` (default: torch's current stream of x's device); nothing is synchronised unless
    check=True (then the device status word is read back and DeviceError raised if set).
    `status`: optional 1-element int32 CUDA tensor the AIRTOPK_ERR_* bits are OR-ed into.
    sorted=True: each row comes out in selection order (one extra launch, K <= 4096).
    """
    torch = _torch()
    if not x.is_cuda:
        raise ValueError("select() needs a CUDA tensor (no CPU fallback)")
    squeeze = x.dim() == 1
    x2 = x.reshape(1, -1) if squeeze else x
    if x2.dim() != 2 or not x2.is_contiguous():
        raise ValueError("x must be a contiguous [batch, len] or [len] tensor")
    batch, length = x2.shape
    dt = dtype_code(x2.dtype)
    dev = x2.device
    # the library queries and launches on the current device: make it x's (skipped when it already
    # is: the context manager costs a few microseconds per call)
    with (_NULLCTX if dev.index == torch.cuda.current_device() else torch.cuda.device(dev)):
        if out is None:
            vals = torch.empty((batch, k), dtype=x2.dtype, device=dev)
            idx = torch.empty((batch, k), dtype=torch.int64, device=dev)
        else:
            vals, idx = out
            _check_out(vals, (batch, k), x2.dtype, dev, "out[0] (values)")
            _check_out(idx, (batch, k), torch.int64, dev, "out[1] (indices)")
        st = _status_word(check, status, dev)
        o = _opts(alpha, engine, ctas_per_row, cluster_size, trace, events, window, tma, early_stop, st, sorted)
        L = lib()
        if workspace is None:
            workspace = _workspace(None, int(L.airtopk_workspace_bytes_ex(dt, batch, length, k, ctypes.byref(o))), dev)
        elif workspace.dtype != torch.uint8 or workspace.device != dev or not workspace.is_contiguous():
            raise ValueError(f"workspace must be a contiguous uint8 tensor on {dev}")
        # (a caller workspace that is too small is rejected by the library: AIRTOPK_ENOSPACE)
        ws_ptr = workspace.data_ptr() if workspace is not None else None
        ws_bytes = workspace.numel() if workspace is not None else 0
        s = _stream(stream, dev)
        _check(L.airtopk_select_ex(x2.data_ptr(), dt, batch, length, k, 0 if largest else 1,
                                   vals.data_ptr(), idx.data_ptr(), ws_ptr, ws_bytes, s, ctypes.byref(o)))
        if check:
            _raise_status(st)
    if squeeze:
        return vals[0], idx[0]
    return vals, idx


def select_with_idx(x, in_idx, k: int, idx_bits: int, largest: bool = False, workspace=None, stream=None,
                    out=None, status=None, check: bool = False, engine: int = ENGINE_AUTO):
    """Merge select over one row whose elements carry index VALUES in_idx (int64, distinct, <
    2^idx_bits); ties rank by in_idx value; returned indices are in_idx values."""
    torch = _torch()
    x = x.reshape(-1)
    in_idx = in_idx.reshape(-1)
    if not (x.is_cuda and in_idx.is_cuda and in_idx.dtype == torch.int64 and in_idx.numel() == x.numel()
            and x.device == in_idx.device and x.is_contiguous() and in_idx.is_contiguous()):
        raise ValueError("select_with_idx: x and in_idx must be contiguous CUDA tensors of equal length "
                         "(in_idx int64) on one device")
    dt = dtype_code(x.dtype)
    n = x.numel()
    dev = x.device
    with torch.cuda.device(dev):
        if out is None:
            vals = torch.empty(k, dtype=x.dtype, device=dev)
            idx = torch.empty(k, dtype=torch.int64, device=dev)
        else:
            vals, idx = out
            _check_out(vals, (k,), x.dtype, dev, "out[0] (values)")
            _check_out(idx, (k,), torch.int64, dev, "out[1] (indices)")
        need = int(lib().airtopk_workspace_bytes_with_idx(dt, n, k, idx_bits))
        workspace = _workspace(workspace, need, dev)
        st = _status_word(check, status, dev)
        o = _opts(engine=engine, status=st)
        _check(lib().airtopk_select_with_idx_ex(x.data_ptr(), in_idx.data_ptr(), idx_bits, dt, n, k,
                                                0 if largest else 1, vals.data_ptr(), idx.data_ptr(),
                                                workspace.data_ptr() if workspace is not None else None,
                                                workspace.numel() if workspace is not None else 0,
                                                _stream(stream, dev), ctypes.byref(o)))
        if check:
            _raise_status(st)
    return vals, idx


def merge_idx_bits(total_len: int, world: int, k: int) -> int:
    """Index width of the split-row merge (global indices and pad indices < total_len + world*k)."""
    b = int(lib().airtopk_merge_idx_bits(total_len, world, k))
    if b <= 0:
        raise ValueError("merge_idx_bits: invalid arguments")
    return b


def select_shard(x_shard, k: int, shard_offset: int, pad_base: int, largest: bool = False, out=None,
                 workspace=None, stream=None):
    """Local step of a split-row select (airtopk_select_shard): exactly k entries — the shard's top
    min(k, len) with GLOBAL indices (local + shard_offset), then pad entries (keys that sort last,
    indices pad_base + j) when the shard is shorter than k. out = (values[k], int64 indices[k])
    may be views into the gather buffers (the all-gather then runs in place)."""
    torch = _torch()
    x = x_shard.reshape(-1)
    if not x.is_cuda or not x.is_contiguous():
        raise ValueError("select_shard needs a contiguous CUDA tensor")
    dt = dtype_code(x.dtype)
    dev = x.device
    n = x.numel()
    with torch.cuda.device(dev):
        if out is None:
            vals = torch.empty(k, dtype=x.dtype, device=dev)
            idx = torch.empty(k, dtype=torch.int64, device=dev)
        else:
            vals, idx = out
            _check_out(vals, (k,), x.dtype, dev, "out[0] (values)")
            _check_out(idx, (k,), torch.int64, dev, "out[1] (indices)")
        need = int(lib().airtopk_workspace_bytes_shard(dt, n, k))
        workspace = _workspace(workspace, need, dev)
        _check(lib().airtopk_select_shard(x.data_ptr(), dt, n, k, 0 if largest else 1, int(shard_offset),
                                          int(pad_base), vals.data_ptr(), idx.data_ptr(),
                                          workspace.data_ptr() if workspace is not None else None,
                                          workspace.numel() if workspace is not None else 0, _stream(stream, dev)))
    return vals, idx


def select_ablation(x, k: int, design: int, digit_bits: int = 11, largest: bool = False, alpha: int = 0):
    """The paper's kernel-organisation ablations (airtopk_select_ablation): design 0 naive (Fig. 2),
    1 iteration-fused (Fig. 3), 2 fused last filter; digit_bits 8 or 11. Returns
    (values, indices, kernel launches)."""
    torch = _torch()
    x2 = x.reshape(1, -1) if x.dim() == 1 else x
    if not x2.is_cuda or not x2.is_contiguous():
        raise ValueError("select_ablation needs a contiguous CUDA tensor")
    batch, length = x2.shape
    dt = dtype_code(x2.dtype)
    dev = x2.device
    with torch.cuda.device(dev):
        vals = torch.empty((batch, k), dtype=x2.dtype, device=dev)
        idx = torch.empty((batch, k), dtype=torch.int64, device=dev)
        need = int(lib().airtopk_ablation_workspace(dt, batch, length, alpha))
        ws = torch.empty(max(need, 1), dtype=torch.uint8, device=dev)
        nk = ctypes.c_int(0)
        _check(lib().airtopk_select_ablation(x2.data_ptr(), dt, batch, length, k, 0 if largest else 1, vals.data_ptr(),
                                             idx.data_ptr(), int(design), int(digit_bits), int(alpha), ws.data_ptr(),
                                             ws.numel(), _stream(None, dev), ctypes.byref(nk)))
    return vals, idx, int(nk.value)


def select_host(x_host, k: int, largest: bool = False, out=None, stream=None):
    """End-to-end select on HOST tensors (pinned for async DMA): H2D, select, D2H, synchronise."""
    torch = _torch()
    if x_host.is_cuda or not x_host.is_contiguous():
        raise ValueError("select_host needs a contiguous host tensor")
    x2 = x_host.reshape(1, -1) if x_host.dim() == 1 else x_host
    batch, length = x2.shape
    dt = dtype_code(x2.dtype)
    if out is None:
        pin = x_host.is_pinned()
        vals = torch.empty((batch, k), dtype=x2.dtype, pin_memory=pin)
        idx = torch.empty((batch, k), dtype=torch.int64, pin_memory=pin)
    else:
        vals, idx = out
        if tuple(vals.shape) != (batch, k) or tuple(idx.shape) != (batch, k) or vals.is_cuda or idx.is_cuda \
                or vals.dtype != x2.dtype or idx.dtype != torch.int64:
            raise ValueError("select_host: out must be host tensors ([batch, k] values, int64 indices)")
    s = (stream if stream is not None else torch.cuda.current_stream()).cuda_stream
    _check(lib().airtopk_select_host(x2.data_ptr(), dt, batch, length, k, 0 if largest else 1,
                                     vals.data_ptr(), idx.data_ptr(), s))
    return vals, idx


def trace_buffer(batch: int, device="cuda"):
    torch = _torch()
    return torch.full((batch, TRACE_MAX_PASSES, 10), -1, dtype=torch.int64, device=device)
