"""B200-native AIR Top-K (Zhang et al., SC'23) — thin Python binding over libairtopk.so.

Every step of the selection runs in the CUDA kernels of libairtopk.so (csrc/); this module only
marshals torch tensors (device memory, the current stream) into the C ABI of include/airtopk.h.
There is no CPU fallback: calling without the built library or on a CPU tensor raises.

    values, indices = select(x, k, largest=False)      # x: [batch, len] or [len] CUDA tensor
"""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import AirTopKError, Options, OK, ENGINE_AUTO, ENGINE_GRID, ENGINE_CLUSTER, ENGINE_GRIDSELECT, TRACE_MAX_PASSES

__all__ = ["select", "select_with_idx", "select_host", "workspace_bytes", "describe", "lib", "AirTopKError",
           "ENGINE_AUTO", "ENGINE_GRID", "ENGINE_CLUSTER", "ENGINE_GRIDSELECT", "dtype_code"]

_LIB = None


def lib():
    """The loaded libairtopk.so (raises ImportError if it was not built)."""
    global _LIB
    if _LIB is None:
        _LIB = _lib.load()
    return _LIB


def _torch():
    import torch
    return torch


def dtype_code(dtype) -> int:
    torch = _torch()
    m = {torch.float32: _lib.F32, torch.float16: _lib.F16, torch.bfloat16: _lib.BF16,
         torch.float64: _lib.F64, torch.uint32: _lib.U32}
    if dtype not in m:
        raise TypeError(f"unsupported key dtype {dtype} (f32/f16/bf16/f64/u32)")
    return m[dtype]


def _check(status: int):
    if status != OK:
        raise AirTopKError(status, lib())


def _opts(alpha=0, engine=ENGINE_AUTO, ctas_per_row=0, cluster_size=0, trace=None, events=None, window=0, tma=0,
          early_stop=0):
    o = Options()
    o.early_stop = int(early_stop)
    o.window = int(window)
    o.tma = int(tma)
    o.alpha = int(alpha)
    o.engine = int(engine)
    o.ctas_per_row = int(ctas_per_row)
    o.cluster_size = int(cluster_size)
    o.trace = trace.data_ptr() if trace is not None else None
    if events is not None:
        # events: a ctypes array of cudaEvent_t handles (see make_event_array)
        o.events = ctypes.cast(events, ctypes.c_void_p)
        o.n_events = len(events)
    return o


def make_event_array(events):
    """ctypes array of the raw cudaEvent_t handles of torch.cuda.Event objects (already created)."""
    arr = (ctypes.c_void_p * len(events))()
    for j, e in enumerate(events):
        arr[j] = e.cuda_event
    return arr


def workspace_bytes(dtype, batch: int, length: int, k: int, alpha: int = 0) -> int:
    o = _opts(alpha)
    return int(lib().airtopk_workspace_bytes_ex(dtype_code(dtype), batch, length, k, ctypes.byref(o)))


def describe(dtype, batch: int, length: int, k: int, alpha: int = 0, engine: int = ENGINE_AUTO,
             ctas_per_row: int = 0, cluster_size: int = 0, window: int = 0, tma: int = 0) -> dict:
    """How a select with these arguments runs: engine, passes, launches, grid shape, workspace."""
    o = _opts(alpha, engine, ctas_per_row, cluster_size, window=window, tma=tma)
    pl = _lib.Plan()
    _check(lib().airtopk_describe(dtype_code(dtype), batch, length, k, ctypes.byref(o), ctypes.byref(pl)))
    return {f: getattr(pl, f) for f, _ in _lib.Plan._fields_}


def select(x, k: int, largest: bool = False, *, alpha: int = 0, engine: int = ENGINE_AUTO,
           ctas_per_row: int = 0, cluster_size: int = 0, trace=None, events=None, window: int = 0,
           tma: int = 0, early_stop: int = 0, workspace=None, out=None, stream=None):
    """Top-K of each row of `x` ([batch, len] or [len], contiguous CUDA tensor).

    Returns (values, indices): [batch, k] of x.dtype (raw bit copies) and int64 row-local indices,
    order within a row unspecified. Ties at the K-th value go to the lowest index. Enqueued on
    `stream` (default: torch's current stream); nothing is synchronised.
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
    if out is None:
        vals = torch.empty((batch, k), dtype=x2.dtype, device=x2.device)
        idx = torch.empty((batch, k), dtype=torch.int64, device=x2.device)
    else:
        vals, idx = out
    o = _opts(alpha, engine, ctas_per_row, cluster_size, trace, events, window, tma, early_stop)
    need = int(lib().airtopk_workspace_bytes_ex(dt, batch, length, k, ctypes.byref(o)))
    if workspace is None and need:
        workspace = torch.empty(need, dtype=torch.uint8, device=x2.device)
    ws_ptr = workspace.data_ptr() if workspace is not None else None
    ws_bytes = workspace.numel() if workspace is not None else 0
    s = (stream if stream is not None else torch.cuda.current_stream(x2.device)).cuda_stream
    _check(lib().airtopk_select_ex(x2.data_ptr(), dt, batch, length, k, 0 if largest else 1,
                                   vals.data_ptr(), idx.data_ptr(), ws_ptr, ws_bytes, s, ctypes.byref(o)))
    if squeeze:
        return vals[0], idx[0]
    return vals, idx


def select_with_idx(x, in_idx, k: int, idx_bits: int, largest: bool = False, workspace=None, stream=None):
    """Merge select over one row whose elements carry index VALUES in_idx (int64, distinct, <
    2^idx_bits); ties rank by in_idx value; returned indices are in_idx values."""
    torch = _torch()
    x = x.reshape(-1)
    in_idx = in_idx.reshape(-1)
    assert x.is_cuda and in_idx.is_cuda and in_idx.dtype == torch.int64 and in_idx.numel() == x.numel()
    assert x.is_contiguous() and in_idx.is_contiguous()
    dt = dtype_code(x.dtype)
    n = x.numel()
    vals = torch.empty(k, dtype=x.dtype, device=x.device)
    idx = torch.empty(k, dtype=torch.int64, device=x.device)
    need = int(lib().airtopk_workspace_bytes_with_idx(dt, n, k, idx_bits))
    if workspace is None:
        workspace = torch.empty(max(need, 1), dtype=torch.uint8, device=x.device)
    s = (stream if stream is not None else torch.cuda.current_stream(x.device)).cuda_stream
    _check(lib().airtopk_select_with_idx(x.data_ptr(), in_idx.data_ptr(), idx_bits, dt, n, k,
                                         0 if largest else 1, vals.data_ptr(), idx.data_ptr(),
                                         workspace.data_ptr(), workspace.numel(), s))
    return vals, idx


def select_host(x_host, k: int, largest: bool = False, out=None, stream=None):
    """End-to-end select on HOST tensors (pinned for async DMA): H2D, select, D2H, synchronise."""
    torch = _torch()
    assert not x_host.is_cuda and x_host.is_contiguous()
    x2 = x_host.reshape(1, -1) if x_host.dim() == 1 else x_host
    batch, length = x2.shape
    dt = dtype_code(x2.dtype)
    if out is None:
        pin = x_host.is_pinned()
        vals = torch.empty((batch, k), dtype=x2.dtype, pin_memory=pin)
        idx = torch.empty((batch, k), dtype=torch.int64, pin_memory=pin)
    else:
        vals, idx = out
    s = (stream if stream is not None else torch.cuda.current_stream()).cuda_stream
    _check(lib().airtopk_select_host(x2.data_ptr(), dt, batch, length, k, 0 if largest else 1,
                                     vals.data_ptr(), idx.data_ptr(), s))
    return vals, idx


def trace_buffer(batch: int, device="cuda"):
    torch = _torch()
    return torch.full((batch, TRACE_MAX_PASSES, 10), -1, dtype=torch.int64, device=device)
