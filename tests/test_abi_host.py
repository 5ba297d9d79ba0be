"""Host-side checks of the C-ABI library (no GPU): it loads, exports every symbol include/locassm.h
declares, and its host helpers follow the paper's sizing rule."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_awanhedbdoy21_b200 import build, _lib
    build.build()
    return _lib.load()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "locassm.h")).read()
    return sorted(set(re.findall(r"^\s*(?:la_status|const char \*|int64_t|double)\s*\*?\s*(la_\w+)\s*\(", src, re.M)))


def test_exports_every_declared_symbol(lib):
    names = declared_symbols()
    assert set(names) >= {"la_create", "la_load_batch", "la_extend", "la_destroy"}
    for n in names:
        assert hasattr(lib, n), n


def test_load_factor_helper(lib):
    """P1: table size l*r for (l-k+1)*r k-mers -> load factor (l-k+1)/l; 0.93 at (300, 21)."""
    assert abs(lib.la_paper_load_factor(300, 21) - 280 / 300) < 1e-12
    assert round(lib.la_paper_load_factor(300, 21), 2) == 0.93


def test_global_capacity_bound(lib):
    """The global-table capacity keeps the load factor <= 0.7 even if every insert is distinct."""
    for n in (0, 1, 117, 5000, 10 ** 6, 5 * 10 ** 7):
        cap = lib.la_plan_global_capacity(n)
        assert cap >= n + 1 and n <= 0.7 * cap + 1e-9


def test_no_gpu_create_fails_cleanly(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    c = ctypes.c_void_p()
    assert lib.la_create(ctypes.byref(c), 0, None) == -3
    assert lib.la_destroy(None) == 0


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_awanhedbdoy21_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", txt).replace("oracle/", ""), f


def test_append_extensions_null_context(lib):
    """la_append_extensions rejects a NULL context without touching the device."""
    lib.la_append_extensions.argtypes = [ctypes.c_void_p, ctypes.c_int32] + [ctypes.c_void_p] * 6
    lib.la_append_extensions.restype = ctypes.c_int
    assert lib.la_append_extensions(None, 0, None, None, None, None, None, None) == -1


def test_c_client_builds_and_links(lib):
    """examples/abi_client.c is a plain C99 client of include/locassm.h: it compiles against the header
    alone and its binary resolves liblocassm.so (it is run against a GPU in test_gpu_parity.py)."""
    import subprocess
    import sys
    sys.path.insert(0, ROOT)
    import __graft_entry__
    __graft_entry__.build()
    exe = os.path.join(ROOT, "examples", "abi_client")
    assert os.path.exists(exe)
    out = subprocess.run(["ldd", exe], capture_output=True, text=True).stdout
    assert "liblocassm.so" in out and "not found" not in out


def test_api_rejects_wrong_dtypes(lib):
    """The binding refuses arrays the C library would misread (int32 offsets, non-byte sequences)."""
    import numpy as np
    from gen import cases as C  # noqa: F401  (input layout only)
    from paper_conf_sc_awanhedbdoy21_b200.api import _ptr_and_mem
    with pytest.raises(ValueError):
        _ptr_and_mem(np.zeros(3, np.int32), "read_off", "int64")
    with pytest.raises(ValueError):
        _ptr_and_mem(np.zeros(3, np.int64), "read_seq", "bytes")
    assert _ptr_and_mem(np.zeros(3, np.int64), "read_off", "int64")[1] is False
