"""CPU correctness oracle for AIR Top-K — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference` legs may
import this package. The product package (paper_conf_sc_zhangnlw23_b200) never imports it and
shares no code with it (see oracle.cpp's header for the definitions and paper citations).

Every function takes numpy arrays and returns canonical results sorted by (code, index).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

DT = {np.dtype(np.float32): 0, np.dtype(np.float16): 1, "bfloat16": 2, np.dtype(np.float64): 3,
      np.dtype(np.uint32): 4}
DT_NAMES = {"f32": 0, "f16": 1, "bf16": 2, "f64": 3, "u32": 4}


def build(force: bool = False) -> str:
    """Compile the oracle (plain C++17, -O2; OpenMP only in oracle_topk_nth_mt, the all-cores
    CPU baseline variant — every other function is single-threaded)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-std=c++17", "-O2", "-fopenmp", "-fPIC", "-shared", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i64, vp, ci = ctypes.c_int64, ctypes.c_void_p, ctypes.c_int
        for name in ("oracle_topk_sort", "oracle_topk_nth", "oracle_topk_brute"):
            f = getattr(lib, name)
            f.argtypes = [ci, vp, i64, i64, i64, ci, vp, vp]
            f.restype = ci
        lib.oracle_topk_nth_mt.argtypes = [ci, vp, i64, i64, i64, ci, vp, vp, ctypes.POINTER(ci)]
        lib.oracle_topk_nth_mt.restype = ci
        lib.oracle_topk_with_idx.argtypes = [ci, vp, vp, i64, i64, ci, vp, vp]
        lib.oracle_topk_with_idx.restype = ci
        lib.oracle_codes.argtypes = [ci, vp, i64, ci, vp]
        lib.oracle_codes.restype = ci
        lib.oracle_rbits.argtypes = [ci]
        lib.oracle_rbits.restype = ci
        lib.oracle_radix_trace.argtypes = [vp, i64, ci, ci, ci, i64, i64, ci, vp, vp, vp, ci]
        lib.oracle_radix_trace.restype = ci
        _lib = lib
    return _lib


def dtype_code(arr_or_name) -> int:
    if isinstance(arr_or_name, str):
        return DT_NAMES[arr_or_name]
    return DT[np.dtype(arr_or_name.dtype)]


def _prep(keys: np.ndarray, dt):
    keys = np.ascontiguousarray(keys)
    if keys.ndim == 1:
        keys = keys[None, :]
    if dt is None:
        dt = dtype_code(keys)
    return keys, dt


def _run(fname, keys, k, select_min=True, dt=None):
    keys, dt = _prep(keys, dt)
    batch, n = keys.shape
    vals = np.empty((batch, k), dtype=keys.dtype)
    idx = np.empty((batch, k), dtype=np.int64)
    rc = getattr(_L(), fname)(dt, keys.ctypes.data, batch, n, k, int(bool(select_min)),
                              vals.ctypes.data, idx.ctypes.data)
    if rc != 0:
        raise ValueError(f"{fname} failed rc={rc} (batch={batch} len={n} k={k})")
    return vals, idx


def topk_sort(keys, k, select_min=True, dt=None):
    """(values, indices) of the K smallest (largest) per row; canonical (code, idx) order."""
    return _run("oracle_topk_sort", keys, k, select_min, dt)


def topk_nth(keys, k, select_min=True, dt=None):
    return _run("oracle_topk_nth", keys, k, select_min, dt)


def topk_nth_mt(keys, k, select_min=True, dt=None):
    """All-cores variant (OpenMP chunks + candidate merge). Returns (values, indices, threads)."""
    keys, dt = _prep(keys, dt)
    batch, n = keys.shape
    vals = np.empty((batch, k), dtype=keys.dtype)
    idx = np.empty((batch, k), dtype=np.int64)
    th = ctypes.c_int(0)
    rc = _L().oracle_topk_nth_mt(dt, keys.ctypes.data, batch, n, k, int(bool(select_min)),
                                 vals.ctypes.data, idx.ctypes.data, ctypes.byref(th))
    if rc != 0:
        raise ValueError(f"oracle_topk_nth_mt failed rc={rc}")
    return vals, idx, int(th.value)


def topk_brute(keys, k, select_min=True, dt=None):
    return _run("oracle_topk_brute", keys, k, select_min, dt)


topk = topk_nth


def topk_with_idx(keys, in_idx, k, select_min=True, dt=None):
    keys, dt = _prep(keys, dt)
    keys = keys.reshape(-1)
    in_idx = np.ascontiguousarray(in_idx, dtype=np.int64).reshape(-1)
    assert in_idx.size == keys.size
    vals = np.empty(k, dtype=keys.dtype)
    idx = np.empty(k, dtype=np.int64)
    rc = _L().oracle_topk_with_idx(dt, keys.ctypes.data, in_idx.ctypes.data, keys.size, k,
                                   int(bool(select_min)), vals.ctypes.data, idx.ctypes.data)
    if rc != 0:
        raise ValueError(f"oracle_topk_with_idx rc={rc}")
    return vals, idx


def codes(keys, select_min=True, dt=None) -> np.ndarray:
    """Order-preserving codes, same shape as `keys` (uint64)."""
    shape = np.shape(keys)
    keys, dt = _prep(keys, dt)
    flat = keys.reshape(-1)
    out = np.empty(flat.size, dtype=np.uint64)
    rc = _L().oracle_codes(dt, flat.ctypes.data, flat.size, int(bool(select_min)), out.ctypes.data)
    if rc != 0:
        raise ValueError("bad dtype")
    return out.reshape(shape)


def rbits(dt) -> int:
    return int(_L().oracle_rbits(dt if isinstance(dt, int) else dtype_code(dt)))


TRACE_FIELDS = ("width", "src_L", "stored", "j", "K", "C", "Cp", "emitted", "early_stop", "read")


def radix_trace(code_arr, k, r_bits=32, b=11, idx_bits=0, alpha=128, early_stop=True):
    """Algorithm 1 step by step on one row of codes (uint64). Returns (sel_idx, records, hists)
    where records is a list of dicts (one per kernel, the last one being the final emission)."""
    c = np.ascontiguousarray(code_arr, dtype=np.uint64).reshape(-1)
    n = c.size
    maxrec = -(-r_bits // b) + -(-idx_bits // b) + 1
    sel = np.empty(k, dtype=np.int64)
    tr = np.zeros((maxrec, 10), dtype=np.int64)
    hist = np.zeros((maxrec, 1 << b), dtype=np.int64)
    rc = _L().oracle_radix_trace(c.ctypes.data, n, r_bits, b, idx_bits, k, alpha, int(bool(early_stop)),
                                 sel.ctypes.data, tr.ctypes.data, hist.ctypes.data, maxrec)
    if rc < 0:
        raise ValueError(f"oracle_radix_trace rc={rc}")
    recs = [dict(zip(TRACE_FIELDS, map(int, tr[i]))) for i in range(rc)]
    return sel, recs, hist[: rc - 1]
