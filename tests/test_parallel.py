"""Multi-GPU driver host logic, CPU only.

The shard split and the result gather are exercised with world_size-2 gloo
process groups on CPU tensors; the per-rank scores are the oracle's, so no
GPU is needed.  The CUDA side of the same driver runs in
tests/test_gpu_parity.py::test_multi_device_driver and in bench.py --gpus N.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_ipps_nishimurabin17_b200 import parallel


@pytest.mark.parametrize("P", [0, 1, 31, 32, 33, 1000, 1024, 4097, 1 << 20])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_shard_ranges_partition(P, world):
    rs = parallel.shard_ranges(P, world)
    assert rs[0][0] == 0 and rs[-1][1] == P
    for (a, b), (c, d) in zip(rs, rs[1:]):
        assert b == c  # contiguous, disjoint
    sizes = [b - a for a, b in rs]
    assert all(s >= 0 for s in sizes)
    # 32-pair-group granular: every boundary except the end is a multiple of 32
    assert all(a % 32 == 0 or a == P for a, _ in rs)
    groups = [(b - a + 31) // 32 for a, b in rs]
    assert max(groups) - min(groups) <= 1


def test_shard_range_rejects_bad_args():
    with pytest.raises(ValueError):
        parallel.shard_range(10, 0, 0)
    with pytest.raises(ValueError):
        parallel.shard_range(10, 2, 2)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, P, m, n, seed, result_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        b, e = parallel.shard_range(P, world, rank)
        # each rank regenerates only its shard (global pair index p_offset)
        q, t = synth.gen_pairs(seed, e - b, m, n, planted=True, p_offset=b)
        local = torch.from_numpy(oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))
        full = parallel.gather_scores(local, P)
        if rank == 0:
            np.save(result_path, full.numpy())
        dist.barrier()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P", [1000, 64, 33])
def test_gloo_gather_reassembles_global_batch(tmp_path, P):
    world, m, n, seed = 2, 24, 40, 1234
    path = str(tmp_path / "full.npy")
    mp.spawn(_worker, args=(world, _free_port(), P, m, n, seed, path), nprocs=world, join=True)
    full = np.load(path)
    q, t = synth.gen_pairs(seed, P, m, n, planted=True)
    np.testing.assert_array_equal(full, oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))


def _worker_uneven(rank, world, port, result_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        P = 32 * 3 + 5  # 4 groups over 2 ranks: 64 + 37 pairs
        b, e = parallel.shard_range(P, world, rank)
        local = torch.arange(b, e, dtype=torch.int32) * 7
        full = parallel.gather_scores(local, P)
        bad = None
        try:
            parallel.gather_scores(local[:-1], P) if e > b else None
        except ValueError as exc:
            bad = str(exc)
        if rank == 0:
            np.save(result_path, full.numpy())
            assert bad is not None
    finally:
        dist.destroy_process_group()


def test_gloo_gather_uneven_shards(tmp_path):
    path = str(tmp_path / "u.npy")
    mp.spawn(_worker_uneven, args=(2, _free_port(), path), nprocs=2, join=True)
    np.testing.assert_array_equal(np.load(path), np.arange(101, dtype=np.int32) * 7)


def _worker_c3(rank, world, port, result_path):
    """bench.py's strong-scaled C3 path on CPU (BASELINE configs[2]: 2^22
    pairs sharded over the ranks): each rank generates only its
    shard_range shard (p_offset), scores it (the oracle stands in for the
    device here), the int32 scores are all-gathered over gloo, and rank 0
    checks bench.py's 65 536-pair parity sample, regenerated from global pair
    indices, against the gathered scores.  Lengths are cut to 4 x 5 so the
    2^22 pairs stay cheap on the CPU; the pair count and the shard split are
    C3's."""
    import bench
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        P_total, m, n, seed = bench.CONFIGS[3]["P"], 4, 5, synth.seed_for_config(3)
        b, e = parallel.shard_range(P_total, world, rank)
        assert e - b == P_total // world  # 2^22 splits evenly over 2 ranks
        q, t = synth.gen_pairs(seed, e - b, m, n, p_offset=b)
        local = torch.from_numpy(oracle.sw_batch(q, t, 2, -1, -1, score_bits=4))
        full = parallel.gather_scores(local, P_total).numpy()
        if rank == 0:
            idx = bench.gathered_sample_index(P_total, m)
            qs, ts = bench.regen_pairs(seed, idx, m, n)
            want = oracle.sw_batch(qs, ts, 2, -1, -1, score_bits=4)
            np.save(result_path, np.array([idx.size, int((full[idx] != want).sum()),
                                           full.size], dtype=np.int64))
        dist.barrier()
    finally:
        dist.destroy_process_group()


def test_gloo_c3_strong_shards_and_bench_parity_sample(tmp_path):
    path = str(tmp_path / "c3.npy")
    mp.spawn(_worker_c3, args=(2, _free_port(), path), nprocs=2, join=True)
    k, mism, total = np.load(path)
    assert (k, mism, total) == (65536, 0, 1 << 22)
