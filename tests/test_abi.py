"""C-ABI library checks that need no GPU: it loads, exports every function
include/bpbc_sw.h declares (with the binding's signatures), and its host-only
entry points validate arguments.  Also checks that the product never reaches
the oracle."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_ipps_nishimurabin17_b200 as bpbc
from paper_conf_ipps_nishimurabin17_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bpbc_sw.h")
PKG = os.path.join(ROOT, "paper_conf_ipps_nishimurabin17_b200")


def header_functions():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^(?:int|const char \*)\s*(bpbc_sw_\w+)\(", src, re.M)))


def test_library_exports_every_declared_symbol():
    names = header_functions()
    assert len(names) >= 10
    lib = _lib.load()
    for nm in names:
        assert hasattr(lib, nm), nm
    assert sorted(_lib.SIGNATURES) == names
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True,
                         text=True).stdout
    for nm in names:
        assert re.search(rf"\bT {nm}$", out, re.M), nm


def test_status_strings():
    lib = _lib.load()
    for code in range(-5, 1):
        s = lib.bpbc_sw_status_string(code).decode()
        assert s and s != "unknown status"
    assert lib.bpbc_sw_status_string(-99).decode() == "unknown status"


def test_workspace_bytes_host_only():
    # planes 8 B per position per 32-pair group + padding + partial maxima
    P, m, n = 1 << 20, 128, 128
    b = bpbc.workspace_bytes(P, m, n)
    G = P // 32
    assert b >= 8 * G * (m + n) + G * 32 * 16 * 4
    assert b < 8 * G * (m + n) + G * 32 * 16 * 4 + (1 << 20)
    assert bpbc.workspace_bytes(P, n, m) == b            # symmetric
    assert bpbc.workspace_bytes(0, 5, 7) > 0
    with pytest.raises(bpbc.BPBCError):
        bpbc.workspace_bytes(-1, 5, 7)
    with pytest.raises(bpbc.BPBCError):
        bpbc.workspace_bytes(10, 0, 7)


def test_null_ctx_and_bad_args_rejected():
    lib = _lib.load()
    assert lib.bpbc_sw_score_batch(None, None, None, 10, 5, 5, 2, -1, -1, 8, None, None, 0,
                                   None) == _lib.BPBC_ERR_INVALID_ARG
    assert lib.bpbc_sw_init(0, None) == _lib.BPBC_ERR_INVALID_ARG
    assert lib.bpbc_sw_destroy(None) == _lib.BPBC_OK
    assert lib.bpbc_sw_get_error_flags(None, None) == _lib.BPBC_ERR_INVALID_ARG


def test_init_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    lib = _lib.load()
    c = ctypes.c_void_p()
    rc = lib.bpbc_sw_init(0, ctypes.byref(c))
    assert rc in (_lib.BPBC_ERR_CUDA, _lib.BPBC_ERR_INVALID_ARG)
    assert not c.value


def test_product_never_imports_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", src, re.M), f
                assert "sw_oracle" not in src, f
    deps = subprocess.run(["ldd", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "oracle" not in deps


def test_binding_fails_loudly_without_library(tmp_path, monkeypatch):
    monkeypatch.setattr(_lib, "LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(_lib, "_lib", None)
    with pytest.raises(ImportError):
        _lib.load()
