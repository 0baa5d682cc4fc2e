"""synth -- seeded synthetic inputs shared by the oracle side and the CUDA side.

Holds none of the method's arithmetic: it only draws DNA base codes
A=0, T=1, G=2, C=3 (the paper's A=00, T=01, G=10, C=11) with a
counter-based SplitMix64, so any shard of any batch can be regenerated
independently (pair index p is global, ``p_offset`` shifts a shard).

Recipe: i.i.d. uniform bases, matching the paper's
random-like workloads of fixed lengths m, n; ``planted=True`` adds the
parity-test stream where 1/64 of pairs have target = query tiled to length n
and 1/16 have a 10%-substituted copy, which drives scores to the width cap.

``gen_pairs`` uses the C implementation (synth/gen.c, threads); ``gen_pairs_np``
is the readable numpy definition it is tested against.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB = os.path.join(_HERE, "_build", "libsynth.so")
_lock = threading.Lock()
_lib = None

# Seeds of BASELINE.json configs: 0xB9BC0000 + config id.
SEED_BASE = 0xB9BC0000

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def build(force: bool = False) -> str:
    os.makedirs(os.path.dirname(_LIB), exist_ok=True)
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            lib.synth_gen_pairs.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64,
                                            ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
            lib.synth_gen_pairs.restype = ctypes.c_int
            _lib = lib
    return _lib


def gen_pairs(seed: int, num_pairs: int, m: int, n: int, planted: bool = False,
              p_offset: int = 0, out_q: np.ndarray | None = None,
              out_t: np.ndarray | None = None, threads: int | None = None):
    """Return (q uint8 [P][m], t uint8 [P][n]).  out_q/out_t may be given
    (e.g. numpy views of pinned host tensors) to fill in place."""
    q = out_q if out_q is not None else np.empty((num_pairs, m), dtype=np.uint8)
    t = out_t if out_t is not None else np.empty((num_pairs, n), dtype=np.uint8)
    assert q.shape == (num_pairs, m) and t.shape == (num_pairs, n)
    assert q.flags.c_contiguous and t.flags.c_contiguous
    if num_pairs:
        _load().synth_gen_pairs(seed & 0xFFFFFFFFFFFFFFFF, num_pairs, p_offset, m, n,
                                int(planted), q.ctypes.data, t.ctypes.data,
                                threads or os.cpu_count() or 1)
    return q, t


def _mix(z: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = z + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def gen_pairs_np(seed: int, num_pairs: int, m: int, n: int, planted: bool = False,
                 p_offset: int = 0):
    """Readable numpy definition of gen_pairs (small sizes only)."""
    s = np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
    p = (np.arange(num_pairs, dtype=np.uint64) + np.uint64(p_offset))[:, None]
    i = np.arange(m, dtype=np.uint64)[None, :]
    j = np.arange(n, dtype=np.uint64)[None, :]
    q = (_mix(s ^ (p << np.uint64(24)) ^ i) >> np.uint64(62)).astype(np.uint8)
    t = (_mix(s ^ np.uint64(1 << 63) ^ (p << np.uint64(24)) ^ j) >> np.uint64(62)).astype(np.uint8)
    if planted:
        sel = _mix(s ^ np.uint64(3 << 62) ^ p[:, 0])
        exact = (sel & np.uint64(63)) == 1
        mut = ((sel & np.uint64(15)) == 0) & ~exact
        tiled = q[:, np.arange(n) % m]
        h = _mix(s ^ np.uint64(1 << 62) ^ (p << np.uint64(24)) ^ j)
        sub = (h % np.uint64(10)) == 0
        subst = ((tiled.astype(np.uint64) + np.uint64(1) + (h >> np.uint64(62)) % np.uint64(3))
                 & np.uint64(3)).astype(np.uint8)
        mutated = np.where(sub, subst, tiled)
        t = np.where(exact[:, None], tiled, t)
        t = np.where(mut[:, None], mutated, t)
    return np.ascontiguousarray(q), np.ascontiguousarray(t)


def seed_for_config(config_id: int) -> int:
    return SEED_BASE + config_id


def encode(s: str) -> np.ndarray:
    """'ATGC' string -> codes (A=0, T=1, G=2, C=3)."""
    table = {"A": 0, "T": 1, "G": 2, "C": 3}
    return np.array([table[c] for c in s.upper()], dtype=np.uint8)


def pack2bit(codes: np.ndarray) -> np.ndarray:
    """Input-format helper (no method arithmetic): uint8 codes [P, len] ->
    2-bit packed rows [P, ceil(len/4)], base i in bits 2(i%4) of byte i//4
    (the layout of bpbc_sw_score_batch_packed2, include/bpbc_sw.h)."""
    codes = np.asarray(codes, dtype=np.uint8)
    P, ln = codes.shape
    w = (ln + 3) // 4
    pad = np.zeros((P, 4 * w), dtype=np.uint8)
    pad[:, :ln] = codes & 3
    q = pad.reshape(P, w, 4)
    return np.ascontiguousarray(q[:, :, 0] | (q[:, :, 1] << 2) | (q[:, :, 2] << 4) | (q[:, :, 3] << 6))


def unpack2bit(packed: np.ndarray, ln: int) -> np.ndarray:
    """Inverse of pack2bit."""
    packed = np.asarray(packed, dtype=np.uint8)
    P = packed.shape[0]
    out = np.stack([(packed >> (2 * k)) & 3 for k in range(4)], axis=2).reshape(P, -1)
    return np.ascontiguousarray(out[:, :ln])
