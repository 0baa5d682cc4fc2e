"""Multi-GPU driver: shard independent pair batches over devices / ranks.

The BPBC batch is embarrassingly parallel: pairs are independent and all have
the same lengths, so the work per 32-pair group is identical.
The driver therefore splits the ceil(P/32) groups into contiguous ranges, one
per device, runs the whole hot path (pack -> sweep -> extract) on each device
with its own ctx and stream, and has NO collective on the data path
(DESIGN.md section 7).  The only cross-device traffic is the
optional final gather of the int32 scores (4 B per pair).

Two drivers:
  * ``score_sharded`` -- one process per GPU under torch.distributed (NCCL on
    GPUs); each rank scores its shard, ``gather_scores`` optionally
    all-gathers the results;
  * ``score_multi_device`` -- one process, one host thread per device, host
    buffers in and out (the paper's Steps 1-5 per shard).
"""
from __future__ import annotations

import threading

import numpy as np
import torch

from . import api


def shard_range(num_pairs: int, world: int, rank: int) -> tuple[int, int]:
    """Pair range [begin, end) of ``rank`` out of ``world``: contiguous,
    32-pair-group granular, sizes differ by at most one group; ranks past
    the last group get an empty range."""
    if world < 1 or not 0 <= rank < world or num_pairs < 0:
        raise ValueError("bad world/rank/num_pairs")
    groups = (num_pairs + 31) // 32
    base, rem = divmod(groups, world)
    g0 = rank * base + min(rank, rem)
    g1 = g0 + base + (1 if rank < rem else 0)
    return min(num_pairs, 32 * g0), min(num_pairs, 32 * g1)


def shard_ranges(num_pairs: int, world: int) -> list[tuple[int, int]]:
    return [shard_range(num_pairs, world, r) for r in range(world)]


def gather_scores(local: torch.Tensor, num_pairs: int, group=None) -> torch.Tensor:
    """All-gather every rank's int32 shard (``shard_range`` layout) into one
    [num_pairs] tensor on every rank.  Shards are padded to the largest shard
    for ``all_gather_into_tensor`` and trimmed after.  Works with NCCL (CUDA
    tensors) and gloo (CPU tensors)."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    ranges = shard_ranges(num_pairs, world)
    b, e = ranges[rank]
    if local.numel() != e - b:
        raise ValueError(f"rank {rank}: local shard has {local.numel()} scores, expected {e - b}")
    width = max(hi - lo for lo, hi in ranges) if ranges else 0
    buf = torch.zeros(width, dtype=torch.int32, device=local.device)
    buf[: local.numel()] = local
    allbuf = torch.empty(world * width, dtype=torch.int32, device=local.device)
    if hasattr(dist, "all_gather_into_tensor") and local.device.type == "cuda":
        dist.all_gather_into_tensor(allbuf, buf, group=group)
    else:
        parts = list(allbuf.view(world, width).unbind(0)) if width else [allbuf] * world
        dist.all_gather(parts, buf, group=group)
    out = torch.empty(num_pairs, dtype=torch.int32, device=local.device)
    for r, (lo, hi) in enumerate(ranges):
        out[lo:hi] = allbuf[r * width: r * width + (hi - lo)]
    return out


def score_sharded(query: torch.Tensor, target: torch.Tensor, num_pairs: int, match: int = 2,
                  mismatch: int = -1, gap: int = -1, score_bits: int | None = None,
                  gather: bool = False, workspace: torch.Tensor | None = None,
                  stream=None, group=None) -> torch.Tensor:
    """Score this rank's shard under torch.distributed.

    ``query`` / ``target`` hold ONLY this rank's pairs (rows
    ``shard_range(num_pairs, world, rank)`` of the global batch) on this
    rank's CUDA device.  Returns the local int32 scores, or with
    ``gather=True`` the global [num_pairs] scores on every rank."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    b, e = shard_range(num_pairs, world, rank)
    if query.shape[0] != e - b or target.shape[0] != e - b:
        raise ValueError(f"rank {rank}: expected {e - b} local pairs, got {query.shape[0]}")
    if e > b:
        local = api.score_batch(query, target, match, mismatch, gap, score_bits=score_bits,
                                workspace=workspace, stream=stream)
    else:
        local = torch.empty(0, dtype=torch.int32, device=query.device)
    return gather_scores(local, num_pairs, group) if gather else local


def score_multi_device(query: np.ndarray, target: np.ndarray, match: int = 2,
                       mismatch: int = -1, gap: int = -1, score_bits: int | None = None,
                       devices: list[int] | None = None,
                       out: np.ndarray | None = None, return_flags: bool = False):
    """Host arrays in, host int32 scores out, sharded over ``devices`` (one
    host thread per device, each with its own ctx that is destroyed when the
    thread ends, running the blocking host-buffer C call on its slice).  A
    failing shard raises with its device id.  return_flags=True also returns
    each shard's sticky error flags (bit 0 = a base code > 3)."""
    query = np.ascontiguousarray(query, dtype=np.uint8)
    target = np.ascontiguousarray(target, dtype=np.uint8)
    P, m = query.shape
    n = target.shape[1]
    if score_bits is None:
        score_bits = api.default_score_bits(match, m, n)
    if devices is None:
        devices = list(range(torch.cuda.device_count()))
    if not devices:
        raise RuntimeError("score_multi_device: no CUDA device")
    if out is None:
        out = np.empty(P, dtype=np.int32)
    errors: dict[int, BaseException] = {}
    flags = [0] * len(devices)

    def work(rank, dev):
        b, e = shard_range(P, len(devices), rank)
        if e <= b:
            return
        try:
            api.score_batch_host(query[b:e], target[b:e], match, mismatch, gap, score_bits,
                                 device=dev, out=out[b:e])
            flags[rank] = api.get_error_flags(dev)
        except BaseException as exc:  # re-raised below with the device id
            errors[dev] = exc
        finally:
            # this thread's ctx (and its shard-sized device buffers) ends with it
            api.release_thread_ctx(dev)

    threads = [threading.Thread(target=work, args=(r, d)) for r, d in enumerate(devices)]
    for t in threads:
        t.start()
    for t in threads:
        t.join()
    if errors:
        dev, exc = next(iter(errors.items()))
        raise RuntimeError(f"shard on cuda:{dev} failed: {exc}") from exc
    if return_flags:
        return out, flags
    return out
