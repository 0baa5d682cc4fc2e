"""Python binding of the BPBC Smith-Waterman C ABI (include/bpbc_sw.h).

Same names as the C entry points; torch is used for device memory and
streams only.  Every step of the path (pack, sweep, max reduction,
untranspose) runs in the CUDA kernels of libbpbc_sw.so.
"""
from __future__ import annotations

import ctypes
import threading

import numpy as np
import torch

from . import _lib
from ._lib import check

_ctx_lock = threading.Lock()
_ctxs: dict[tuple[int, int], ctypes.c_void_p] = {}


def _ctx(device: int) -> ctypes.c_void_p:
    """The calling thread's ctx for ``device`` (a ctx is not thread-safe:
    one per device per host thread, include/bpbc_sw.h)."""
    key = (device, threading.get_ident())
    with _ctx_lock:
        c = _ctxs.get(key)
        if c is None:
            c = ctypes.c_void_p()
            check(_lib.load().bpbc_sw_init(device, ctypes.byref(c)))
            _ctxs[key] = c
        return c


def destroy_all() -> None:
    with _ctx_lock:
        for c in _ctxs.values():
            _lib.load().bpbc_sw_destroy(c)
        _ctxs.clear()


def release_thread_ctx(device: int) -> None:
    """Destroy the calling thread's ctx for ``device`` (worker threads call
    this before they exit, so their device buffers do not outlive them)."""
    key = (device, threading.get_ident())
    with _ctx_lock:
        c = _ctxs.pop(key, None)
    if c is not None:
        _lib.load().bpbc_sw_destroy(c)


def default_score_bits(match: int, m: int, n: int) -> int:
    """s = bit_length(match * min(m, n)) (reading R2), in [4, 16]."""
    return min(16, max(4, (match * min(m, n)).bit_length()))


def _stream_ptr(stream, device) -> int:
    if stream is None:
        stream = torch.cuda.current_stream(device)
    return stream.cuda_stream


def workspace_bytes(num_pairs: int, m: int, n: int) -> int:
    """bpbc_sw_workspace_bytes: upper bound over every plan of these sizes."""
    v = ctypes.c_size_t()
    check(_lib.load().bpbc_sw_workspace_bytes(num_pairs, m, n, ctypes.byref(v)))
    return v.value


def workspace_bytes_for(num_pairs: int, m: int, n: int, match: int = 2, mismatch: int = -1,
                        gap: int = -1, score_bits: int | None = None, filter: bool = False,
                        device: int = 0) -> int:
    """bpbc_sw_workspace_bytes_for: the exact workspace of that call on ``device``."""
    if score_bits is None:
        score_bits = default_score_bits(match, m, n)
    v = ctypes.c_size_t()
    ctx = _ctx(device)
    check(_lib.load().bpbc_sw_workspace_bytes_for(ctx, num_pairs, m, n, match, mismatch, gap,
                                                  score_bits, int(bool(filter)),
                                                  ctypes.byref(v)), ctx)
    return v.value


def score_batch(query: torch.Tensor, target: torch.Tensor, match: int = 2, mismatch: int = -1,
                gap: int = -1, score_bits: int | None = None, out: torch.Tensor | None = None,
                workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """bpbc_sw_score_batch on CUDA tensors query uint8 [P, m], target uint8 [P, n].

    Returns int32 [P] = min(max local score, 2^score_bits - 1), enqueued on
    ``stream`` (default: torch's current stream of the tensors' device)."""
    if not (query.is_cuda and target.is_cuda):
        raise ValueError("score_batch needs CUDA tensors (use score_batch_host for host arrays)")
    if query.dtype != torch.uint8 or target.dtype != torch.uint8:
        raise TypeError("query/target must be uint8 base codes")
    if query.dim() != 2 or target.dim() != 2 or query.shape[0] != target.shape[0]:
        raise ValueError("query [P, m] and target [P, n] expected")
    query, target = query.contiguous(), target.contiguous()
    P, m = query.shape
    n = target.shape[1]
    dev = query.device.index if query.device.index is not None else torch.cuda.current_device()
    if score_bits is None:
        score_bits = default_score_bits(match, m, n)
    if out is None:
        out = torch.empty(P, dtype=torch.int32, device=query.device)
    ws_ptr, ws_bytes = None, 0
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    ctx = _ctx(dev)
    check(_lib.load().bpbc_sw_score_batch(ctx, query.data_ptr(), target.data_ptr(), P, m, n, match,
                                          mismatch, gap, score_bits, out.data_ptr(), ws_ptr,
                                          ws_bytes, _stream_ptr(stream, query.device)), ctx)
    return out


def score_batch_host(query: np.ndarray, target: np.ndarray, match: int = 2, mismatch: int = -1,
                     gap: int = -1, score_bits: int | None = None, device: int = 0,
                     out: np.ndarray | None = None) -> np.ndarray:
    """bpbc_sw_score_batch_host: host arrays in, host int32 scores out (blocking).
    ``query``/``target`` may be numpy views of pinned torch tensors."""
    query = np.ascontiguousarray(query, dtype=np.uint8)
    target = np.ascontiguousarray(target, dtype=np.uint8)
    P, m = query.shape
    n = target.shape[1]
    if score_bits is None:
        score_bits = default_score_bits(match, m, n)
    if out is None:
        out = np.empty(P, dtype=np.int32)
    ctx = _ctx(device)
    check(_lib.load().bpbc_sw_score_batch_host(ctx, query.ctypes.data, target.ctypes.data, P, m, n,
                                               match, mismatch, gap, score_bits, out.ctypes.data),
          ctx)
    return out


def filter_batch(query: torch.Tensor, target: torch.Tensor, threshold: int, match: int = 2,
                 mismatch: int = -1, gap: int = -1, score_bits: int | None = None,
                 indices: bool = True, workspace: torch.Tensor | None = None,
                 stream=None):
    """bpbc_sw_filter_batch: flag the pairs whose max local score > threshold
    (the paper's filter use case).

    Returns (mask, count, idx): mask int32 [ceil(P/32)] CUDA tensor of flag
    words (bit k of word g = pair 32g+k; int32 view of the uint32 words),
    count an int64 [1] CUDA tensor, idx an int64 [P] CUDA tensor whose first
    count entries are the flagged pairs in ascending order (None if
    indices=False)."""
    if not (query.is_cuda and target.is_cuda):
        raise ValueError("filter_batch needs CUDA tensors")
    if query.dtype != torch.uint8 or target.dtype != torch.uint8:
        raise TypeError("query/target must be uint8 base codes")
    if query.dim() != 2 or target.dim() != 2 or query.shape[0] != target.shape[0]:
        raise ValueError("query [P, m] and target [P, n] expected")
    query, target = query.contiguous(), target.contiguous()
    P, m = query.shape
    n = target.shape[1]
    dev = query.device.index if query.device.index is not None else torch.cuda.current_device()
    if score_bits is None:
        score_bits = default_score_bits(match, m, n)
    # outputs are allocated on the stream the C call writes them on (the C
    # side writes every count / mask word, no zero fill needed)
    st = stream if stream is not None else torch.cuda.current_stream(query.device)
    with torch.cuda.stream(st):
        mask = torch.empty((P + 31) // 32, dtype=torch.int32, device=query.device)
        count = torch.empty(1, dtype=torch.int64, device=query.device)
        idx = torch.empty(P, dtype=torch.int64, device=query.device) if indices else None
    ws_ptr, ws_bytes = None, 0
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    ctx = _ctx(dev)
    check(_lib.load().bpbc_sw_filter_batch(
        ctx, query.data_ptr(), target.data_ptr(), P, m, n, match, mismatch, gap, score_bits,
        threshold, mask.data_ptr(), idx.data_ptr() if idx is not None else None,
        count.data_ptr(), ws_ptr, ws_bytes, st.cuda_stream), ctx)
    return mask, count, idx


def score_batch_wordwise(query: torch.Tensor, target: torch.Tensor, match: int = 2,
                         mismatch: int = -1, gap: int = -1, out: torch.Tensor | None = None,
                         workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """bpbc_sw_score_batch_wordwise: the wordwise (non-bitwise) 16-bit SIMD
    comparator on the same inputs; exact int32 scores (no width cap)."""
    if not (query.is_cuda and target.is_cuda):
        raise ValueError("score_batch_wordwise needs CUDA tensors")
    if query.dtype != torch.uint8 or target.dtype != torch.uint8:
        raise TypeError("query/target must be uint8 base codes")
    query, target = query.contiguous(), target.contiguous()
    P, m = query.shape
    n = target.shape[1]
    dev = query.device.index if query.device.index is not None else torch.cuda.current_device()
    if out is None:
        out = torch.empty(P, dtype=torch.int32, device=query.device)
    ws_ptr, ws_bytes = None, 0
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    ctx = _ctx(dev)
    check(_lib.load().bpbc_sw_score_batch_wordwise(
        ctx, query.data_ptr(), target.data_ptr(), P, m, n, match, mismatch, gap, out.data_ptr(),
        ws_ptr, ws_bytes, _stream_ptr(stream, query.device)), ctx)
    return out


def score_batch_packed2(query2: torch.Tensor, target2: torch.Tensor, m: int, n: int,
                        match: int = 2, mismatch: int = -1, gap: int = -1,
                        score_bits: int | None = None, out: torch.Tensor | None = None,
                        workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """bpbc_sw_score_batch_packed2: query2 uint8 [P, ceil(m/4)], target2 uint8
    [P, ceil(n/4)] CUDA tensors of 2-bit packed bases (4 per byte, base i in
    bits 2(i%4) of byte i//4; include/bpbc_sw.h)."""
    if not (query2.is_cuda and target2.is_cuda):
        raise ValueError("score_batch_packed2 needs CUDA tensors")
    if query2.dtype != torch.uint8 or target2.dtype != torch.uint8:
        raise TypeError("packed rows must be uint8")
    P = query2.shape[0]
    if (query2.shape != (P, (m + 3) // 4) or target2.shape != (P, (n + 3) // 4)):
        raise ValueError("query2 [P, ceil(m/4)] and target2 [P, ceil(n/4)] expected")
    query2, target2 = query2.contiguous(), target2.contiguous()
    dev = query2.device.index if query2.device.index is not None else torch.cuda.current_device()
    if score_bits is None:
        score_bits = default_score_bits(match, m, n)
    if out is None:
        out = torch.empty(P, dtype=torch.int32, device=query2.device)
    ws_ptr, ws_bytes = None, 0
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    ctx = _ctx(dev)
    check(_lib.load().bpbc_sw_score_batch_packed2(
        ctx, query2.data_ptr(), target2.data_ptr(), P, m, n, match, mismatch, gap, score_bits,
        out.data_ptr(), ws_ptr, ws_bytes, _stream_ptr(stream, query2.device)), ctx)
    return out


def score_batch_host_packed2(query2: np.ndarray, target2: np.ndarray, m: int, n: int,
                             match: int = 2, mismatch: int = -1, gap: int = -1,
                             score_bits: int | None = None, device: int = 0,
                             out: np.ndarray | None = None) -> np.ndarray:
    """bpbc_sw_score_batch_host_packed2: host 2-bit packed rows in, host int32
    scores out (blocking; 4x fewer host->device bytes than score_batch_host)."""
    query2 = np.ascontiguousarray(query2, dtype=np.uint8)
    target2 = np.ascontiguousarray(target2, dtype=np.uint8)
    P = query2.shape[0]
    if query2.shape != (P, (m + 3) // 4) or target2.shape != (P, (n + 3) // 4):
        raise ValueError("query2 [P, ceil(m/4)] and target2 [P, ceil(n/4)] expected")
    if score_bits is None:
        score_bits = default_score_bits(match, m, n)
    if out is None:
        out = np.empty(P, dtype=np.int32)
    ctx = _ctx(device)
    check(_lib.load().bpbc_sw_score_batch_host_packed2(
        ctx, query2.ctypes.data, target2.ctypes.data, P, m, n, match, mismatch, gap, score_bits,
        out.ctypes.data), ctx)
    return out


def pack(codes: torch.Tensor, stream=None, out: torch.Tensor | None = None) -> torch.Tensor:
    """bpbc_sw_pack: uint8 [P, len] -> uint32 [ceil(P/32), len, 2] bit planes (H, L)
    (returned as an int32 view; ``out`` may supply that tensor)."""
    codes = codes.contiguous()
    P, ln = codes.shape
    G = (P + 31) // 32
    if out is not None:
        if out.shape != (G, ln, 2) or out.dtype != torch.int32 or not out.is_contiguous():
            raise ValueError(f"out must be a contiguous int32 [{G}, {ln}, 2] tensor")
        planes = out
    else:
        planes = torch.empty((G, ln, 2), dtype=torch.int32, device=codes.device)
    dev = codes.device.index or 0
    ctx = _ctx(dev)
    check(_lib.load().bpbc_sw_pack(ctx, codes.data_ptr(), P, ln, planes.data_ptr(),
                                   _stream_ptr(stream, codes.device)), ctx)
    return planes


def untranspose(partial: torch.Tensor, num_pairs: int, cap: int, stream=None) -> torch.Tensor:
    """bpbc_sw_untranspose: uint32 [G, lanes, s] bit-sliced partial maxima ->
    int32 [num_pairs] = min(max over lanes, cap)."""
    partial = partial.contiguous()
    G, lanes, s = partial.shape
    out = torch.empty(num_pairs, dtype=torch.int32, device=partial.device)
    dev = partial.device.index or 0
    ctx = _ctx(dev)
    check(_lib.load().bpbc_sw_untranspose(ctx, partial.data_ptr(), G, lanes, s, num_pairs, cap,
                                          out.data_ptr(), _stream_ptr(stream, partial.device)), ctx)
    return out


def get_error_flags(device: int = 0) -> int:
    """bpbc_sw_get_error_flags: the sticky flags since the last read (bit 0 =
    BPBC_FLAG_BAD_BASE), cleared.  The C call returns BPBC_ERR_BAD_BASE when
    that bit is set; here the bit is returned (check_flags raises)."""
    v = ctypes.c_uint32()
    ctx = _ctx(device)
    rc = _lib.load().bpbc_sw_get_error_flags(ctx, ctypes.byref(v))
    if rc not in (_lib.BPBC_OK, _lib.BPBC_ERR_BAD_BASE):
        check(rc, ctx)
    return v.value


def check_flags(device: int = 0) -> None:
    """Raise BPBCError(BPBC_ERR_BAD_BASE) if a base code > 3 was seen."""
    if get_error_flags(device) & _lib.BPBC_FLAG_BAD_BASE:
        raise _lib.BPBCError(_lib.BPBC_ERR_BAD_BASE, "a base code > 3 was read as c & 3")


def last_plan(device: int = 0) -> dict:
    """Circuit / width / tiling of the last sweep dispatched on ``device``."""
    c, w, r, l, o = (ctypes.c_int32() for _ in range(5))
    s = ctypes.c_int64()
    check(_lib.load().bpbc_sw_last_plan(_ctx(device), ctypes.byref(c), ctypes.byref(w),
                                        ctypes.byref(r), ctypes.byref(l), ctypes.byref(s),
                                        ctypes.byref(o)))
    k, f = ctypes.c_int32(), ctypes.c_int32()
    check(_lib.load().bpbc_sw_last_launches(_ctx(device), ctypes.byref(k), ctypes.byref(f)))
    wr, bps, hs = ctypes.c_int32(), ctypes.c_int64(), ctypes.c_int32()
    check(_lib.load().bpbc_sw_last_schedule(_ctx(device), ctypes.byref(wr), ctypes.byref(bps),
                                            ctypes.byref(hs)))
    return {"circuit": ["exact", "saturating"][c.value] if c.value >= 0 else None,
            "width": w.value, "rows_per_lane": r.value, "lanes": l.value,
            "streams": s.value, "ops_per_word_cell": o.value, "kernels": k.value,
            "fused": bool(f.value), "wrap": bool(wr.value), "blocks_per_sm": bps.value,
            "host_streamed": bool(hs.value)}


def profile(enable: bool, device: int = 0) -> None:
    """bpbc_sw_profile: start (clearing) / stop per-phase event recording."""
    check(_lib.load().bpbc_sw_profile(_ctx(device), int(bool(enable))))


def profile_read(device: int = 0) -> dict:
    """bpbc_sw_profile_read: summed ms per phase (Table IV columns W2B, SWA,
    B2W) over the calls recorded since the last read; resets."""
    ms = (ctypes.c_double * 4)()
    calls = ctypes.c_int64()
    ctx = _ctx(device)
    check(_lib.load().bpbc_sw_profile_read(ctx, ms, ctypes.byref(calls)), ctx)
    return {"w2b_ms": ms[0], "swa_ms": ms[1], "b2w_ms": ms[2], "total_ms": ms[3],
            "calls": calls.value}
