"""ctypes loader of libbpbc_sw.so (the C ABI of include/bpbc_sw.h).

Argument marshalling only.  The library is built in-tree by
``__graft_entry__.build()`` (``make -C paper_conf_ipps_nishimurabin17_b200/csrc``);
if it is missing, importing the package's compute API fails loudly -- there
is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# BPBC_SW_LIB overrides the library path (benchmark experiments with
# alternative builds only; the in-tree build is the default).
LIB_PATH = os.environ.get("BPBC_SW_LIB") or os.path.join(_HERE, "libbpbc_sw.so")

BPBC_OK = 0
BPBC_ERR_INVALID_ARG = -1
BPBC_ERR_UNSUPPORTED = -2
BPBC_ERR_CUDA = -3
BPBC_ERR_OOM = -4
BPBC_ERR_BAD_BASE = -5
BPBC_FLAG_BAD_BASE = 0x1
BPBC_FLAG_STALL = 0x2

# name -> (restype, argtypes); must match include/bpbc_sw.h
_c = ctypes
_vp = _c.c_void_p
SIGNATURES = {
    "bpbc_sw_init": (_c.c_int, [_c.c_int, _c.POINTER(_vp)]),
    "bpbc_sw_destroy": (_c.c_int, [_vp]),
    "bpbc_sw_workspace_bytes": (_c.c_int, [_c.c_int64, _c.c_int32, _c.c_int32,
                                           _c.POINTER(_c.c_size_t)]),
    "bpbc_sw_workspace_bytes_for": (_c.c_int, [_vp, _c.c_int64, _c.c_int32, _c.c_int32,
                                               _c.c_int32, _c.c_int32, _c.c_int32, _c.c_int32,
                                               _c.c_int32, _c.POINTER(_c.c_size_t)]),
    "bpbc_sw_score_batch": (_c.c_int, [_vp, _vp, _vp, _c.c_int64, _c.c_int32, _c.c_int32,
                                       _c.c_int32, _c.c_int32, _c.c_int32, _c.c_int32, _vp,
                                       _vp, _c.c_size_t, _vp]),
    "bpbc_sw_score_batch_host": (_c.c_int, [_vp, _vp, _vp, _c.c_int64, _c.c_int32,
                                            _c.c_int32, _c.c_int32, _c.c_int32, _c.c_int32,
                                            _c.c_int32, _vp]),
    "bpbc_sw_score_batch_packed2": (_c.c_int, [_vp, _vp, _vp, _c.c_int64, _c.c_int32,
                                               _c.c_int32, _c.c_int32, _c.c_int32, _c.c_int32,
                                               _c.c_int32, _vp, _vp, _c.c_size_t, _vp]),
    "bpbc_sw_score_batch_host_packed2": (_c.c_int, [_vp, _vp, _vp, _c.c_int64, _c.c_int32,
                                                    _c.c_int32, _c.c_int32, _c.c_int32,
                                                    _c.c_int32, _c.c_int32, _vp]),
    "bpbc_sw_filter_batch": (_c.c_int, [_vp, _vp, _vp, _c.c_int64, _c.c_int32, _c.c_int32,
                                        _c.c_int32, _c.c_int32, _c.c_int32, _c.c_int32,
                                        _c.c_int32, _vp, _vp, _vp, _vp, _c.c_size_t, _vp]),
    "bpbc_sw_wordwise_workspace_bytes": (_c.c_int, [_c.c_int64, _c.POINTER(_c.c_size_t)]),
    "bpbc_sw_score_batch_wordwise": (_c.c_int, [_vp, _vp, _vp, _c.c_int64, _c.c_int32,
                                                _c.c_int32, _c.c_int32, _c.c_int32, _c.c_int32,
                                                _vp, _vp, _c.c_size_t, _vp]),
    "bpbc_sw_pack": (_c.c_int, [_vp, _vp, _c.c_int64, _c.c_int32, _vp, _vp]),
    "bpbc_sw_untranspose": (_c.c_int, [_vp, _vp, _c.c_int64, _c.c_int32, _c.c_int32,
                                       _c.c_int64, _c.c_int32, _vp, _vp]),
    "bpbc_sw_get_error_flags": (_c.c_int, [_vp, _c.POINTER(_c.c_uint32)]),
    "bpbc_sw_last_plan": (_c.c_int, [_vp, _c.POINTER(_c.c_int32), _c.POINTER(_c.c_int32),
                                     _c.POINTER(_c.c_int32), _c.POINTER(_c.c_int32),
                                     _c.POINTER(_c.c_int64), _c.POINTER(_c.c_int32)]),
    "bpbc_sw_last_launches": (_c.c_int, [_vp, _c.POINTER(_c.c_int32), _c.POINTER(_c.c_int32)]),
    "bpbc_sw_last_schedule": (_c.c_int, [_vp, _c.POINTER(_c.c_int32), _c.POINTER(_c.c_int64),
                                         _c.POINTER(_c.c_int32)]),
    "bpbc_sw_profile": (_c.c_int, [_vp, _c.c_int]),
    "bpbc_sw_profile_read": (_c.c_int, [_vp, _c.POINTER(_c.c_double), _c.POINTER(_c.c_int64)]),
    "bpbc_sw_status_string": (_c.c_char_p, [_c.c_int]),
    "bpbc_sw_last_error": (_c.c_char_p, [_vp]),
}

_lib = None


def load() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(
                f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'` "
                "(the CUDA path has no CPU fallback)")
        lib = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(lib, name)
            fn.restype = res
            fn.argtypes = args
        _lib = lib
    return _lib


class BPBCError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        msg = load().bpbc_sw_status_string(status).decode()
        super().__init__(f"bpbc_sw status {status} ({msg}){': ' + detail if detail else ''}")


def check(status: int, ctx=None) -> None:
    if status != BPBC_OK:
        detail = ""
        if ctx is not None and status in (BPBC_ERR_CUDA, BPBC_ERR_OOM):
            detail = load().bpbc_sw_last_error(ctx).decode()
        raise BPBCError(status, detail)
