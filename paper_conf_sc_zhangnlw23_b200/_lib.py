"""ctypes binding of libairtopk.so (include/airtopk.h). Argument marshalling only.

There is deliberately no fallback: if the CUDA library is missing the import fails loudly.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AIRTOPK_LIB", os.path.join(_PKG, "libairtopk.so"))

OK, EINVAL, EDTYPE, ENOSPACE, ECUDA, EDEVICE = 0, 1, 2, 3, 4, 5
ERR_OUTPUT_OVERFLOW, ERR_BUFFER_OVERFLOW, ERR_COUNT = 1, 2, 4
F32, F16, BF16, F64, U32 = 0, 1, 2, 3, 4
ENGINE_AUTO, ENGINE_GRID, ENGINE_CLUSTER, ENGINE_GRIDSELECT, ENGINE_BATCH, ENGINE_RESIDENT, ENGINE_GRIDSELECT_PTQ = \
    0, 1, 2, 4, 5, 6, 7
TRACE_MAX_PASSES = 16
TRACE_FIELDS = ("width", "src_L", "stored", "j", "K", "C", "Cp", "emitted", "early_stop", "read")

# Every symbol include/airtopk.h declares (checked by tests/test_abi.py).
EXPORTS = (
    "airtopk_workspace_bytes", "airtopk_workspace_bytes_ex", "airtopk_select", "airtopk_select_ex",
    "airtopk_select_f32", "airtopk_select_f16", "airtopk_select_bf16", "airtopk_select_f64",
    "airtopk_select_u32", "airtopk_workspace_bytes_with_idx", "airtopk_select_with_idx",
    "airtopk_select_host", "airtopk_status_str", "airtopk_last_cuda_error", "airtopk_version",
    "airtopk_describe", "airtopk_select_with_idx_ex", "airtopk_workspace_bytes_shard", "airtopk_select_shard",
    "airtopk_merge_idx_bits", "airtopk_ipc_handle", "airtopk_ipc_open", "airtopk_ipc_close", "airtopk_shard_push",
    "airtopk_wait_flags", "airtopk_ablation_workspace", "airtopk_select_ablation",
)


class Options(ctypes.Structure):
    _fields_ = [
        ("alpha", ctypes.c_int64),
        ("engine", ctypes.c_int32),
        ("ctas_per_row", ctypes.c_int32),
        ("cluster_size", ctypes.c_int32),
        ("n_events", ctypes.c_int32),
        ("trace", ctypes.c_void_p),
        ("events", ctypes.c_void_p),
        ("window", ctypes.c_int32),
        ("tma", ctypes.c_int32),
        ("early_stop", ctypes.c_int32),
        ("status", ctypes.c_void_p),
        ("sorted", ctypes.c_int32),
        ("trace_len", ctypes.c_int64),
    ]


class Plan(ctypes.Structure):
    _fields_ = [
        ("engine", ctypes.c_int32),
        ("passes", ctypes.c_int32),
        ("launches", ctypes.c_int32),
        ("ctas_per_row", ctypes.c_int32),
        ("cluster_size", ctypes.c_int32),
        ("index_bits", ctypes.c_int32),
        ("buffer_cap", ctypes.c_int64),
        ("workspace_bytes", ctypes.c_size_t),
    ]


class AirTopKError(RuntimeError):
    def __init__(self, status: int, lib=None):
        msg = lib.airtopk_status_str(status).decode() if lib is not None else f"status {status}"
        if status == ECUDA and lib is not None:
            msg += f" (cudaError {lib.airtopk_last_cuda_error()})"
        super().__init__(msg)
        self.status = status


class AirTopKArgumentError(AirTopKError, ValueError):
    """AIRTOPK_EINVAL / EDTYPE / ENOSPACE: the call's arguments (e.g. a caller workspace that is too
    small) were rejected before anything was enqueued."""


def load(path: str = LIB_PATH):
    if not os.path.exists(path):
        raise ImportError(f"{path} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                          "or `python -m paper_conf_sc_zhangnlw23_b200._build` (no CPU fallback exists)")
    lib = ctypes.CDLL(path)
    i64, vp, ci, sz = ctypes.c_int64, ctypes.c_void_p, ctypes.c_int, ctypes.c_size_t
    lib.airtopk_workspace_bytes.argtypes = [ci, i64, i64, i64]
    lib.airtopk_workspace_bytes.restype = sz
    lib.airtopk_workspace_bytes_ex.argtypes = [ci, i64, i64, i64, ctypes.POINTER(Options)]
    lib.airtopk_workspace_bytes_ex.restype = sz
    lib.airtopk_select.argtypes = [vp, ci, i64, i64, i64, ci, vp, vp, vp, sz, vp]
    lib.airtopk_select.restype = ci
    lib.airtopk_select_ex.argtypes = [vp, ci, i64, i64, i64, ci, vp, vp, vp, sz, vp, ctypes.POINTER(Options)]
    lib.airtopk_select_ex.restype = ci
    for n in ("airtopk_select_f32", "airtopk_select_f16", "airtopk_select_bf16", "airtopk_select_f64",
              "airtopk_select_u32"):
        getattr(lib, n).argtypes = [vp, i64, i64, i64, ci, vp, vp, vp]
        getattr(lib, n).restype = ci
    lib.airtopk_workspace_bytes_with_idx.argtypes = [ci, i64, i64, ci]
    lib.airtopk_workspace_bytes_with_idx.restype = sz
    lib.airtopk_select_with_idx.argtypes = [vp, vp, ci, ci, i64, i64, ci, vp, vp, vp, sz, vp]
    lib.airtopk_select_with_idx.restype = ci
    lib.airtopk_select_with_idx_ex.argtypes = [vp, vp, ci, ci, i64, i64, ci, vp, vp, vp, sz, vp, ctypes.POINTER(Options)]
    lib.airtopk_select_with_idx_ex.restype = ci
    lib.airtopk_workspace_bytes_shard.argtypes = [ci, i64, i64]
    lib.airtopk_workspace_bytes_shard.restype = sz
    lib.airtopk_select_shard.argtypes = [vp, ci, i64, i64, ci, i64, i64, vp, vp, vp, sz, vp]
    lib.airtopk_select_shard.restype = ci
    lib.airtopk_merge_idx_bits.argtypes = [i64, ci, i64]
    lib.airtopk_merge_idx_bits.restype = ci
    lib.airtopk_ipc_handle.argtypes = [vp, vp, ctypes.POINTER(ctypes.c_uint64)]
    lib.airtopk_ipc_handle.restype = ci
    lib.airtopk_ipc_open.argtypes = [vp, ctypes.c_uint64, ctypes.POINTER(vp)]
    lib.airtopk_ipc_open.restype = ci
    lib.airtopk_ipc_close.argtypes = [vp]
    lib.airtopk_ipc_close.restype = ci
    lib.airtopk_shard_push.argtypes = [vp, vp, i64, ci, ci, ci, vp, vp, vp, ctypes.c_uint32, vp, vp]
    lib.airtopk_shard_push.restype = ci
    lib.airtopk_wait_flags.argtypes = [vp, ci, ctypes.c_uint32, vp]
    lib.airtopk_wait_flags.restype = ci
    lib.airtopk_ablation_workspace.argtypes = [ci, i64, i64, i64]
    lib.airtopk_ablation_workspace.restype = sz
    lib.airtopk_select_ablation.argtypes = [vp, ci, i64, i64, i64, ci, vp, vp, ci, ci, i64, vp, sz, vp,
                                            ctypes.POINTER(ci)]
    lib.airtopk_select_ablation.restype = ci
    lib.airtopk_select_host.argtypes = [vp, ci, i64, i64, i64, ci, vp, vp, vp]
    lib.airtopk_select_host.restype = ci
    lib.airtopk_status_str.argtypes = [ci]
    lib.airtopk_status_str.restype = ctypes.c_char_p
    lib.airtopk_last_cuda_error.restype = ci
    lib.airtopk_version.restype = ctypes.c_char_p
    lib.airtopk_describe.argtypes = [ci, i64, i64, i64, ctypes.POINTER(Options), ctypes.POINTER(Plan)]
    lib.airtopk_describe.restype = ci
    return lib
