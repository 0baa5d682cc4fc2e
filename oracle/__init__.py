"""oracle -- TEST INFRASTRUCTURE ONLY (never imported by the product package).

Plain CPU definitions of what the BPBC Smith-Waterman hot path computes, used
to check the CUDA path element by element.  Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  It shares no code with
``paper_conf_ipps_nishimurabin17_b200`` and neither imports the other.

Citations ``P:Lnnn`` are lines of the paper text.

Functions
---------
sw_score / sw_batch / sw_matrix
    Scalar int32 Smith-Waterman in plain C (``sw_oracle.c``), P:L192-216,
    with out = min(best, 2^s - 1) (reading R3).
brute_local
    Enumeration of every alignment path (no DP), m, n <= 8.
pack_planes
    Definition of the bit-transpose format: word i of plane
    H/L holds bit H/L of character i of the 32 pairs of a group, bit k =
    pair k; codes A=0 (00), T=1 (01), G=2 (10), C=3 (11).
untranspose
    Definition of bit-untranspose: score of pair k is
    sum_b ((M_b >> k) & 1) << b.

Parity pins for every function live in tests/test_oracle.py; none is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sw_oracle.c")
_LIB_PATH = os.path.join(_HERE, "_build", "libsw_oracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile sw_oracle.c with gcc -O2 (no SIMD flags) into oracle/_build/."""
    os.makedirs(os.path.dirname(_LIB_PATH), exist_ok=True)
    if force or not os.path.exists(_LIB_PATH) or (
            os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC)):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared",
                               "-pthread", "-o", tmp, _SRC])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            u8p = ctypes.POINTER(ctypes.c_uint8)
            i32p = ctypes.POINTER(ctypes.c_int32)
            c_int = ctypes.c_int
            lib.oracle_sw_score.argtypes = [u8p, c_int, u8p, c_int, c_int, c_int, c_int]
            lib.oracle_sw_score.restype = c_int
            lib.oracle_brute_local.argtypes = [u8p, c_int, u8p, c_int, c_int, c_int, c_int]
            lib.oracle_brute_local.restype = c_int
            lib.oracle_sw_matrix.argtypes = [u8p, c_int, u8p, c_int, c_int, c_int, c_int, i32p]
            lib.oracle_sw_matrix.restype = None
            lib.oracle_sw_batch.argtypes = [u8p, u8p, ctypes.c_int64, c_int, c_int, c_int,
                                            c_int, c_int, c_int, i32p, c_int]
            lib.oracle_sw_batch.restype = c_int
            _lib = lib
    return _lib


def _u8(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint8))


def _p(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def sw_score(x, y, match: int = 2, mismatch: int = -1, gap: int = -1) -> int:
    """Max local score of one pair (no width cap)."""
    x, y = _u8(x), _u8(y)
    return _load().oracle_sw_score(_p(x, ctypes.c_uint8), len(x), _p(y, ctypes.c_uint8),
                                   len(y), match, mismatch, gap)


def brute_local(x, y, match: int = 2, mismatch: int = -1, gap: int = -1) -> int:
    x, y = _u8(x), _u8(y)
    if len(x) > 8 or len(y) > 8:
        raise ValueError("brute force only for m, n <= 8")
    return _load().oracle_brute_local(_p(x, ctypes.c_uint8), len(x), _p(y, ctypes.c_uint8),
                                      len(y), match, mismatch, gap)


def sw_matrix(x, y, match: int = 2, mismatch: int = -1, gap: int = -1) -> np.ndarray:
    """(m+1) x (n+1) score matrix including the zero borders."""
    x, y = _u8(x), _u8(y)
    d = np.zeros((len(x) + 1, len(y) + 1), dtype=np.int32)
    _load().oracle_sw_matrix(_p(x, ctypes.c_uint8), len(x), _p(y, ctypes.c_uint8), len(y),
                             match, mismatch, gap, _p(d, ctypes.c_int32))
    return d


def sw_batch(q, t, match: int = 2, mismatch: int = -1, gap: int = -1,
             score_bits: int = 0, threads: int | None = None) -> np.ndarray:
    """Scores of P pairs q[P][m], t[P][n]; score_bits > 0 applies min(., 2^s-1)."""
    q, t = _u8(q), _u8(t)
    if q.ndim != 2 or t.ndim != 2 or q.shape[0] != t.shape[0]:
        raise ValueError("q, t must be [P][m], [P][n]")
    P, m = q.shape
    n = t.shape[1]
    out = np.zeros(P, dtype=np.int32)
    if P == 0:
        return out
    if threads is None:
        threads = os.cpu_count() or 1
    _load().oracle_sw_batch(_p(q, ctypes.c_uint8), _p(t, ctypes.c_uint8), P, m, n, match,
                            mismatch, gap, score_bits, _p(out, ctypes.c_int32), threads)
    return out


def pack_planes(codes) -> np.ndarray:
    """Bit-transpose format by definition.

    codes: uint8 [P][len] with values 0..3.  Returns uint32 [G][len][2]
    (G = ceil(P/32)); [g][i][0] = X^H_i, [g][i][1] = X^L_i of group g, i.e.
    bit k is bit H (resp. L) of character i of pair 32g+k.  Pairs past P read
    as code 0.  Written as the plain per-bit definition, one bit at a time.
    """
    codes = _u8(codes)
    P, ln = codes.shape
    G = (P + 31) // 32
    out = np.zeros((G, ln, 2), dtype=np.uint32)
    for p in range(P):
        g, k = divmod(p, 32)
        hi = ((codes[p] >> 1) & 1).astype(np.uint32) << np.uint32(k)
        lo = (codes[p] & 1).astype(np.uint32) << np.uint32(k)
        out[g, :, 0] |= hi
        out[g, :, 1] |= lo
    return out


def untranspose(planes) -> np.ndarray:
    """Bit-untranspose by definition.

    planes: uint32 [G][s] -- plane b of group g holds bit b of the scores of
    its 32 pairs (bit k = pair 32g+k).  Returns int64 [G*32] scores.
    """
    planes = np.asarray(planes, dtype=np.uint32)
    G, s = planes.shape
    out = np.zeros(G * 32, dtype=np.int64)
    for g in range(G):
        for k in range(32):
            v = 0
            for b in range(s):
                v |= ((int(planes[g, b]) >> k) & 1) << b
            out[32 * g + k] = v
    return out
