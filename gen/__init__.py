"""Seeded synthetic inputs (§5.1; §3.2).

This module is the ONLY code shared by the CUDA path's tests/bench and the CPU oracle's
checks. It contains no top-K arithmetic: it draws key arrays from a counter-based hash
(see gen.c for the exact recipe) so any slice (a batch row, a multi-GPU shard) can be
generated independently and bit-identically.

Config seeds: seed_c = 20231112 + c.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB = os.path.join(_HERE, "libgen.so")
_lib = None

SEED_BASE = 20231112


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-ffp-contract=off",
                               _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        u64, i64, vp = ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p
        for name in ("gen_uniform_f32", "gen_normal_f32", "gen_u32", "gen_u64", "gen_uniform_f64"):
            getattr(lib, name).argtypes = [u64, u64, i64, vp]
            getattr(lib, name).restype = None
        lib.gen_adversarial_f32.argtypes = [u64, u64, i64, ctypes.c_int, vp]
        lib.gen_adversarial_f32.restype = None
        lib.gen_num_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _out(n, dtype, out):
    if out is None:
        out = np.empty(n, dtype=dtype)
    assert out.dtype == dtype and out.flags.c_contiguous and out.size == n
    return out


def uniform_f32(seed: int, n: int, offset: int = 0, out=None) -> np.ndarray:
    """uniform (0, 1] float32."""
    out = _out(n, np.float32, out)
    _L().gen_uniform_f32(seed, offset, n, out.ctypes.data)
    return out


def normal_f32(seed: int, n: int, offset: int = 0, out=None) -> np.ndarray:
    """normal(0, 1) float32 via Box-Muller."""
    out = _out(n, np.float32, out)
    _L().gen_normal_f32(seed, offset, n, out.ctypes.data)
    return out


def adversarial_f32(seed: int, n: int, m_bits: int = 20, offset: int = 0, out=None) -> np.ndarray:
    """radix-adversarial: the first M bits of every element equal those of 1.0f."""
    out = _out(n, np.float32, out)
    _L().gen_adversarial_f32(seed, offset, n, m_bits, out.ctypes.data)
    return out


def u32(seed: int, n: int, offset: int = 0, out=None) -> np.ndarray:
    out = _out(n, np.uint32, out)
    _L().gen_u32(seed, offset, n, out.ctypes.data)
    return out


def u64(seed: int, n: int, offset: int = 0, out=None) -> np.ndarray:
    out = _out(n, np.uint64, out)
    _L().gen_u64(seed, offset, n, out.ctypes.data)
    return out


def uniform_f64(seed: int, n: int, offset: int = 0, out=None) -> np.ndarray:
    out = _out(n, np.float64, out)
    _L().gen_uniform_f64(seed, offset, n, out.ctypes.data)
    return out


def num_threads() -> int:
    return int(_L().gen_num_threads())


DISTS = ("uniform", "normal", "adversarial")


def keys(dist: str, seed: int, n: int, offset: int = 0, m_bits: int = 20, out=None) -> np.ndarray:
    """float32 keys of one of the paper's three distributions."""
    if dist == "uniform":
        return uniform_f32(seed, n, offset, out)
    if dist == "normal":
        return normal_f32(seed, n, offset, out)
    if dist == "adversarial":
        return adversarial_f32(seed, n, m_bits, offset, out)
    raise ValueError(dist)


# The five BASELINE.json configs (SURVEY.md §8 shorthand c1..c5).
CONFIGS = {
    "c1": dict(batch=1, n=1 << 16, k=32, dist="uniform", select_min=True),
    "c2": dict(batch=100, n=1 << 20, k=256, dist="normal", select_min=True),
    "c3": dict(batch=1, n=1 << 30, k=1 << 20, dist="uniform", select_min=True),
    "c4": dict(batch=1, n=1 << 28, k=50000, dist="adversarial", select_min=True),
    "c5": dict(batch=1, n=1 << 33, k=1 << 16, dist="uniform", select_min=True, shards=8),
}


def config_seed(name: str) -> int:
    return SEED_BASE + int(name[1:])


def config_keys(name: str, n: int | None = None, batch: int | None = None, out=None) -> np.ndarray:
    """Keys of config `name` as a [batch, n] float32 array (n/batch overridable for scaled cases).

    Rows are consecutive slices of one global stream (row r starts at global index r*n)."""
    c = CONFIGS[name]
    n = c["n"] if n is None else n
    batch = c["batch"] if batch is None else batch
    flat = keys(c["dist"], config_seed(name), batch * n, 0, out=out)
    return flat.reshape(batch, n)
