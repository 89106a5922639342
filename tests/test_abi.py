"""The C-ABI library loads without a GPU, exports every symbol include/airtopk.h declares, and
validates arguments before touching the device (K in [1, N])."""
import ctypes
import os
import re

import pytest

import paper_conf_sc_zhangnlw23_b200 as at
from paper_conf_sc_zhangnlw23_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "airtopk.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(airtopk_[a-z0-9_]+)\s*\(", src)))


def test_header_and_binding_agree():
    assert header_functions() == sorted(_lib.EXPORTS)


def test_every_declared_symbol_is_exported():
    lib = at.lib()
    for name in header_functions():
        assert hasattr(lib, name), name


def test_status_strings_and_version():
    lib = at.lib()
    for s in range(5):
        assert lib.airtopk_status_str(s).decode().startswith("AIRTOPK_")
    assert lib.airtopk_status_str(99)
    assert lib.airtopk_version().decode().count(".") == 2


def test_argument_validation_without_gpu():
    lib = at.lib()
    p = ctypes.c_void_p(16)
    for batch, n, k in ((1, 10, 0), (1, 10, 11), (0, 10, 1), (1, 0, 1), (-1, 5, 1)):
        assert lib.airtopk_select(p, 0, batch, n, k, 1, p, p, p, 1 << 30, None) == _lib.EINVAL
    assert lib.airtopk_select(p, 9, 1, 10, 1, 1, p, p, p, 1 << 30, None) == _lib.EDTYPE
    assert lib.airtopk_select(None, 0, 1, 10, 1, 1, p, p, p, 1 << 30, None) == _lib.EINVAL
    assert lib.airtopk_select_with_idx(p, None, 10, 0, 10, 1, 1, p, p, p, 1 << 30, None) == _lib.EINVAL
    assert lib.airtopk_select_host(p, 0, 1, 10, 11, 1, p, p, None) == _lib.EINVAL


def test_workspace_small_returns_enospace():
    lib = at.lib()
    p = ctypes.c_void_p(256)
    need = lib.airtopk_workspace_bytes(0, 2, 1 << 20, 100)
    assert need > 0
    assert lib.airtopk_select(p, 0, 2, 1 << 20, 100, 1, p, p, p, need - 1, None) == _lib.ENOSPACE


def test_workspace_bounded_by_alpha():
    """Candidate buffers never exceed N/alpha entries: bytes shrink as alpha grows and
    alpha >= N leaves only the per-row state and histograms."""
    lib = at.lib()
    o = lambda a: ctypes.byref(_lib.Options(alpha=a))
    n = 1 << 24
    b128 = lib.airtopk_workspace_bytes_ex(0, 1, n, 10, o(128))
    b4 = lib.airtopk_workspace_bytes_ex(0, 1, n, 10, o(4))
    bn = lib.airtopk_workspace_bytes_ex(0, 1, n, 10, o(n))
    assert bn < b128 < b4
    assert b128 - bn >= 2 * ((n - 1) // 128) * 8          # two buffers of code+index
    assert b128 - bn <= 2 * ((n - 1) // 128 + 8) * 8 + 1024
    assert lib.airtopk_workspace_bytes(0, 1, 1000, 1000) == 0   # K == N needs no workspace


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_zhangnlw23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                s = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", s), f


def test_gridselect_scope_validation_without_gpu():
    """GridSelect (engines 4 and 7) accepts keys of <= 32 bits, len < 2^32, K <= 2048
     and rejects the rest with AIRTOPK_EINVAL before touching the device."""
    lib = at.lib()
    p = ctypes.c_void_p(256)

    def opts(engine):
        o = _lib.Options()
        o.engine = engine
        return ctypes.byref(o)

    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 32, opts(4)) > 0        # f32, K = 32
    assert lib.airtopk_workspace_bytes_ex(1, 3, 1000, 256, opts(4)) > 0          # f16, K = 256
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 2048, opts(4)) > 0      # K = 2048
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 2048, opts(7)) > 0      # per-thread queues
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 2049, opts(4)) == 0     # K > 2048
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 32, opts(8)) == 0       # no engine 8
    assert lib.airtopk_workspace_bytes_ex(3, 1, 1 << 16, 32, opts(4)) == 0       # f64 keys
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 32, opts(3)) == 0       # no engine 3
    assert lib.airtopk_select_ex(p, 3, 1, 100, 10, 1, p, p, p, 1 << 30, None, opts(4)) == _lib.EINVAL


def test_early_stop_option_validation_without_gpu():
    lib = at.lib()
    o = _lib.Options()
    o.early_stop = -1
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 32, ctypes.byref(o)) > 0
    o.early_stop = 2
    assert lib.airtopk_workspace_bytes_ex(0, 1, 1 << 16, 32, ctypes.byref(o)) == 0
