"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, element by
element on the same seeded inputs (bit-exact, integer results).

Small/medium sizes are checked in full; BASELINE.json's full sizes run in the
launch configuration bench.py times and are checked on a seeded sample of
pairs (the oracle scores each sampled pair on its own).
"""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_ipps_nishimurabin17_b200 as bpbc
from paper_conf_ipps_nishimurabin17_b200 import _lib

pytestmark = pytest.mark.gpu

DEV = "cuda:0"


def run(q, t, match=2, mismatch=-1, gap=-1, s=None):
    dq = torch.from_numpy(np.ascontiguousarray(q)).to(DEV)
    dt = torch.from_numpy(np.ascontiguousarray(t)).to(DEV)
    out = bpbc.score_batch(dq, dt, match, mismatch, gap, score_bits=s)
    return out.cpu().numpy()


def check_full(q, t, match=2, mismatch=-1, gap=-1, s=None):
    m, n = q.shape[1], t.shape[1]
    if s is None:
        s = bpbc.default_score_bits(match, m, n)
    got = run(q, t, match, mismatch, gap, s)
    want = oracle.sw_batch(q, t, match, mismatch, gap, score_bits=s)
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, (f"{bad.size}/{len(want)} mismatches (m={m}, n={n}, s={s}, "
                           f"consts={match},{mismatch},{gap}, plan={bpbc.last_plan(0)}); "
                           f"first pair {bad[0]}: got {got[bad[0]]} want {want[bad[0]]}")
    return got


# ---------------------------------------------------------------- configs


def test_c1_full():
    """BASELINE config 1: 1024 pairs, m = n = 64, +2/-1/-1, 8-bit slices."""
    q, t = synth.gen_pairs(synth.seed_for_config(1), 1024, 64, 64, planted=True)
    got = check_full(q, t, s=8)
    assert got.max() == 128  # planted exact copies reach m * match
    assert bpbc.last_plan(0)["circuit"] == "exact"


@pytest.mark.parametrize("P,m,n,s", [(16384, 128, 128, 9), (4096, 256, 256, 10),
                                     (4096, 64, 1024, 8), (8192, 32, 32, 6), (8192, 64, 64, 7)])
def test_config_shapes_full(P, m, n, s):
    q, t = synth.gen_pairs(synth.seed_for_config(10) + m + n, P, m, n, planted=True)
    check_full(q, t, s=s)


def _sampled(cfg_id, P, m, n, s, sample=8192):
    q, t = synth.gen_pairs(synth.seed_for_config(cfg_id), P, m, n, planted=True)
    got = run(q, t, 2, -1, -1, s)
    rng = np.random.default_rng(cfg_id)
    idx = np.sort(rng.choice(P, size=sample, replace=False))
    idx = np.concatenate([idx, [0, P - 1]])
    want = oracle.sw_batch(q[idx], t[idx], 2, -1, -1, score_bits=s)
    np.testing.assert_array_equal(got[idx], want)
    # properties at any size: 0 <= score <= min(2*min(m,n), 2^s-1)
    assert got.min() >= 0 and got.max() <= min(2 * min(m, n), 2 ** s - 1)


def test_c2_full_size_sampled():
    """BASELINE config 2 at full size (2^20 pairs, m=n=128, s=9)."""
    _sampled(2, 1 << 20, 128, 128, 9)


def test_c4_full_size_sampled():
    """BASELINE config 4 at full size (2^20 pairs, m=64, n=1024, s=8)."""
    _sampled(4, 1 << 20, 64, 1024, 8, sample=4096)


def test_c3_full_size_sampled():
    """BASELINE config 3 per-GPU shard at full size (2^22 pairs, m=n=256, s=10)."""
    _sampled(3, 1 << 22, 256, 256, 10, sample=4096)


# ---------------------------------------------------------------- edge cases


@pytest.mark.parametrize("P", [1, 31, 32, 33, 95, 1000])
def test_ragged_pair_counts(P):
    q, t = synth.gen_pairs(77 + P, P, 40, 56, planted=True)
    check_full(q, t)


@pytest.mark.parametrize("m,n", [(1, 1), (1, 9), (9, 1), (3, 300), (17, 5), (33, 33), (63, 65),
                                 (100, 100), (129, 130), (200, 64), (255, 255), (256, 256),
                                 (256, 1000), (64, 2000)])
def test_lengths(m, n):
    q, t = synth.gen_pairs(5000 + m * 131 + n, 200, m, n, planted=True)
    check_full(q, t)


@pytest.mark.parametrize("m,n", [(32, 32), (7, 32), (32, 7), (31, 64), (16, 96), (20, 40)])
@pytest.mark.parametrize("packed2", [False, True])
def test_short_targets_fused(m, n, packed2):
    """Targets shorter than L + 32 whose length is a multiple of 32 take the
    fused kernel (one query build per phase, at the group boundary itself);
    others (n = 40 < 48) the planes kernel.  Both inputs formats."""
    q, t = synth.gen_pairs(5400 + m * 7 + n, 300, m, n, planted=True)
    want = oracle.sw_batch(q, t, 2, -1, -1)
    if packed2:
        dq = torch.from_numpy(synth.pack2bit(q)).to(DEV)
        dt = torch.from_numpy(synth.pack2bit(t)).to(DEV)
        got = bpbc.score_batch_packed2(dq, dt, m, n, 2, -1, -1).cpu().numpy()
    else:
        got = run(q, t)
    np.testing.assert_array_equal(got, want)
    assert bpbc.last_plan(0)["fused"] == (max(m, n) % 32 == 0)


@pytest.mark.parametrize("s", list(range(4, 17)))
def test_every_width_spec_consts(s):
    q, t = synth.gen_pairs(600 + s, 512, 48, 80, planted=True)
    check_full(q, t, s=s)


@pytest.mark.parametrize("consts", [(1, -1, -1), (3, -2, -1), (1, 0, 0), (2, 0, -1), (5, -3, -4),
                                    (2, -3, -2), (1, -1, 0), (4, -1, -2)])
@pytest.mark.parametrize("s", [5, 8, 12])
def test_runtime_constants(consts, s):
    q, t = synth.gen_pairs(700 + s, 300, 37, 61, planted=True)
    c1, mm, g = consts
    if max(c1, -mm, -g) > 2 ** s - 1:
        pytest.skip("constants must fit")
    check_full(q, t, c1, mm, g, s)


@pytest.mark.parametrize("m", [32, 64, 128, 256])
@pytest.mark.parametrize("s", [6, 7, 8, 9, 10, 11, 12])
def test_c5_width_sweep_saturation(m, s):
    """C5-shaped: the width sweep saturates most pairs at small s (R3)."""
    q, t = synth.gen_pairs(synth.seed_for_config(5) + m, 2048, m, m, planted=True)
    got = check_full(q, t, s=s)
    exact = oracle.sw_batch(q, t, 2, -1, -1)
    np.testing.assert_array_equal(got, np.minimum(exact, 2 ** s - 1))


@pytest.mark.parametrize("consts", [(1, -1, -1), (3, -2, -2), (1, -3, -5), (5, -4, -4), (1, 0, 0)])
@pytest.mark.parametrize("m,n", [(20, 40), (64, 200), (128, 128), (200, 230), (33, 1000),
                                 (300, 310), (512, 520), (600, 640)])
def test_exact_circuit_runtime_constants(consts, m, n):
    """Constants other than (+2, -1, -1) with gap >= mismatch penalty run the
    exact offset circuit with per-bit constant masks (12S + 1 LOP3) on every
    kernel family (planes, L = 16, L = 32, R = 8, multi-warp W = 3 / 4,
    sequential stripes)."""
    c1, mm, g = consts
    q, t = synth.gen_pairs(7100 + m + n + c1, 150, m, n, planted=True)
    s = max(4, (c1 * min(m, n)).bit_length())
    check_full(q, t, c1, mm, g, s)
    plan = bpbc.last_plan(0)
    assert plan["circuit"] == "exact"
    assert plan["ops_per_word_cell"] == 12 * plan["width"] + 1


def test_empty_batch_is_noop():
    q = torch.empty((0, 10), dtype=torch.uint8, device=DEV)
    t = torch.empty((0, 12), dtype=torch.uint8, device=DEV)
    out = bpbc.score_batch(q, t)
    assert out.numel() == 0


def test_errors():
    q = torch.zeros((4, 10), dtype=torch.uint8, device=DEV)
    t = torch.zeros((4, 300), dtype=torch.uint8, device=DEV)
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(q, t, 2, -1, -1, score_bits=3)
    assert ei.value.status == _lib.BPBC_ERR_UNSUPPORTED
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(q, t, 0, -1, -1, score_bits=8)
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(q, t, 2, 1, -1, score_bits=8)
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(q, t, 2, -1, -20, score_bits=4)
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG
    big = torch.zeros((4, (1 << 16) + 1), dtype=torch.uint8, device=DEV)  # > BPBC_MAX_QUERY_LEN
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(big, big)
    assert ei.value.status == _lib.BPBC_ERR_UNSUPPORTED
    ws = torch.empty(16, dtype=torch.uint8, device=DEV)
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(q, q, workspace=ws)
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG


def test_caller_workspace_and_stream():
    q, t = synth.gen_pairs(31337, 777, 50, 70, planted=True)
    ws = torch.empty(bpbc.workspace_bytes(777, 50, 70), dtype=torch.uint8, device=DEV)
    st = torch.cuda.Stream(device=DEV)
    dq = torch.from_numpy(q).to(DEV)
    dt = torch.from_numpy(t).to(DEV)
    torch.cuda.synchronize()
    with torch.cuda.stream(st):
        out = bpbc.score_batch(dq, dt, workspace=ws, stream=st)
    st.synchronize()
    np.testing.assert_array_equal(out.cpu().numpy(),
                                  oracle.sw_batch(q, t, 2, -1, -1, score_bits=8))


def test_bad_base_flag():
    q, t = synth.gen_pairs(9, 64, 20, 20)
    bpbc.get_error_flags(0)  # clear
    q2 = q.copy()
    q2[5, 3] = 7  # not a base code: read as 7 & 3 = 3, flagged
    got = run(q2, t, s=8)
    assert bpbc.get_error_flags(0) & _lib.BPBC_FLAG_BAD_BASE
    np.testing.assert_array_equal(got, oracle.sw_batch(q2 & 3, t, 2, -1, -1, score_bits=8))
    run(q, t, s=8)
    assert bpbc.get_error_flags(0) == 0


def test_host_buffer_path():
    q, t = synth.gen_pairs(4242, 3000, 64, 96, planted=True)
    got = bpbc.score_batch_host(q, t, 2, -1, -1, 8)
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=8))


def test_deterministic_and_input_independent_plan():
    q, t = synth.gen_pairs(11, 4096, 128, 128)
    a = run(q, t, s=9)
    b = run(q, t, s=9)
    np.testing.assert_array_equal(a, b)


# ---------------------------------------------------------------- single steps


@pytest.mark.parametrize("P,ln", [(4, 5), (1, 1), (33, 31), (100, 64), (64, 100), (1000, 129),
                                  (257, 1024)])
def test_pack_kernel_matches_definition(P, ln):
    rng = np.random.default_rng(P * 1000 + ln)
    codes = rng.integers(0, 4, size=(P, ln), dtype=np.uint8)
    planes = bpbc.pack(torch.from_numpy(codes).to(DEV)).cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(planes, oracle.pack_planes(codes))


def test_pack_kernel_paper_example():
    """The 4-pair planes of P:L65-79 through the CUDA pack kernel."""
    xs = np.stack([synth.encode(s) for s in ["ATCGA", "TCGAC", "AAAAA", "TTTTT"]])
    ys = np.stack([synth.encode(s) for s in ["AATCGACA"] * 2 + ["AAAAAAAA", "AATTTTTT"]])
    px = bpbc.pack(torch.from_numpy(xs).to(DEV)).cpu().numpy().view(np.uint32)
    py = bpbc.pack(torch.from_numpy(ys).to(DEV)).cpu().numpy().view(np.uint32)
    assert [int(w) for w in px[0, :, 0]] == [0b0000, 0b0010, 0b0011, 0b0001, 0b0010]
    assert [int(w) for w in px[0, :, 1]] == [0b1010, 0b1011, 0b1001, 0b1000, 0b1010]
    assert [int(w) for w in py[0, :, 0]] == [0, 0, 0, 0b0011, 0b0011, 0, 0b0011, 0]
    assert [int(w) for w in py[0, :, 1]] == [0, 0, 0b1011, 0b1011, 0b1000, 0b1000, 0b1011, 0b1000]


@pytest.mark.parametrize("lanes,s", [(1, 4), (16, 9), (32, 10), (33, 16), (64, 8), (100, 12)])
def test_untranspose_kernel(lanes, s):
    rng = np.random.default_rng(lanes * 100 + s)
    G = 37
    vals = rng.integers(0, 2 ** s, size=(G, lanes, 32))
    partial = np.zeros((G, lanes, s), dtype=np.uint32)
    for b in range(s):
        partial[:, :, b] = (((vals >> b) & 1).astype(np.uint64) << np.arange(32, dtype=np.uint64)
                            ).sum(axis=2).astype(np.uint32)
    cap = 2 ** s - 1 - 3
    P = G * 32 - 5
    got = bpbc.untranspose(torch.from_numpy(partial.view(np.int32)).to(DEV), P, cap).cpu().numpy()
    want = np.minimum(vals.max(axis=1).reshape(-1), cap)[:P]
    np.testing.assert_array_equal(got, want)
    # the definition in the oracle agrees on the reduced planes
    red = np.zeros((G, s), dtype=np.uint32)
    mx = vals.max(axis=1)
    for b in range(s):
        red[:, b] = (((mx >> b) & 1).astype(np.uint64) << np.arange(32, dtype=np.uint64)
                     ).sum(axis=1).astype(np.uint32)
    np.testing.assert_array_equal(np.minimum(oracle.untranspose(red), cap)[:P], want)


def test_multi_device_driver():
    """score_multi_device shards over host threads (here twice cuda:0, one ctx
    per thread) and reassembles; ragged P so shards differ in size."""
    from paper_conf_ipps_nishimurabin17_b200 import parallel
    q, t = synth.gen_pairs(2024, 3001, 64, 80, planted=True)
    got = parallel.score_multi_device(q, t, 2, -1, -1, 8, devices=[0, 0, 0])
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=8))


# ---------------------------------------------------------------- long queries (striped kernel)


@pytest.mark.parametrize("m,n", [(257, 257), (300, 300), (384, 520), (385, 400), (512, 512),
                                 (700, 1000), (1000, 700), (129, 3000), (640, 640)])
def test_long_query_lengths(m, n):
    """min(m, n) > 256: 128-row stripes handed over through the boundary buffer."""
    q, t = synth.gen_pairs(9000 + m * 7 + n, 100, m, n, planted=True)
    check_full(q, t)
    if min(m, n) > 256:
        assert bpbc.last_plan(0)["rows_per_lane"] == 4
    if 256 < min(m, n) <= 512:  # multi-warp: one warp per 128 rows (W = 2..4)
        assert bpbc.last_plan(0)["lanes"] == 32 * ((min(m, n) + 127) // 128)


@pytest.mark.parametrize("s", [6, 8, 10, 11, 12, 16])
def test_c5_m512_width_sweep(s):
    """C5's longest point (m = n = 512) at several widths: saturation law (R3)."""
    q, t = synth.gen_pairs(synth.seed_for_config(5) + 512, 256, 512, 512, planted=True)
    got = check_full(q, t, s=s)
    exact = oracle.sw_batch(q, t, 2, -1, -1)
    np.testing.assert_array_equal(got, np.minimum(exact, 2 ** s - 1))


@pytest.mark.parametrize("consts", [(1, -1, -1), (3, -2, -1), (1, 0, 0), (5, -3, -4)])
def test_long_query_runtime_constants(consts):
    q, t = synth.gen_pairs(4321, 130, 300, 333, planted=True)
    c1, mm, g = consts
    check_full(q, t, c1, mm, g, 12)


@pytest.mark.parametrize("s", [13, 14, 16])
def test_m256_wide_width_uses_stripes(s):
    """m in (128, 256] whose evaluated width is >= 13 bits (match = 31) goes to
    the striped kernel (R = 8 rows x 13+ planes would spill)."""
    q, t = synth.gen_pairs(777 + s, 200, 200, 240, planted=True)
    check_full(q, t, 31, -1, -1, s=s)
    assert bpbc.last_plan(0)["rows_per_lane"] == 4


# ---------------------------------------------------------------- 2-bit packed input (NEXT-1)


@pytest.mark.parametrize("m,n", [(64, 64), (128, 128), (40, 56), (1, 9), (77, 300), (300, 520),
                                 (256, 256)])
def test_packed2_device_matches_oracle(m, n):
    q, t = synth.gen_pairs(6060 + m + n, 999, m, n, planted=True)
    q2 = torch.from_numpy(synth.pack2bit(q)).to(DEV)
    t2 = torch.from_numpy(synth.pack2bit(t)).to(DEV)
    got = bpbc.score_batch_packed2(q2, t2, m, n, 2, -1, -1).cpu().numpy()
    s = bpbc.default_score_bits(2, m, n)
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=s))


def test_packed2_host_matches_u8_path():
    q, t = synth.gen_pairs(7070, 70000, 128, 128, planted=True)  # several host chunks
    got = bpbc.score_batch_host_packed2(synth.pack2bit(q), synth.pack2bit(t), 128, 128, 2, -1, -1, 9)
    ref = bpbc.score_batch_host(q, t, 2, -1, -1, 9)
    np.testing.assert_array_equal(got, ref)
    idx = np.arange(0, 70000, 97)
    np.testing.assert_array_equal(got[idx], oracle.sw_batch(q[idx], t[idx], 2, -1, -1, score_bits=9))


# ---------------------------------------------------------------- threshold filter (NEXT-2)


def _check_filter(q, t, tau, match=2, mismatch=-1, gap=-1, s=None):
    m, n = q.shape[1], t.shape[1]
    if s is None:
        s = bpbc.default_score_bits(match, m, n)
    dq = torch.from_numpy(np.ascontiguousarray(q)).to(DEV)
    dt = torch.from_numpy(np.ascontiguousarray(t)).to(DEV)
    mask, count, idx = bpbc.filter_batch(dq, dt, tau, match, mismatch, gap, score_bits=s)
    P = q.shape[0]
    exact = oracle.sw_batch(q, t, match, mismatch, gap)  # uncapped scores
    want = np.nonzero(exact > tau)[0]
    words = mask.cpu().numpy().view(np.uint32)
    bits = ((words[:, None] >> np.arange(32, dtype=np.uint32)[None, :]) & 1).reshape(-1)[:P]
    np.testing.assert_array_equal(np.nonzero(bits)[0], want)
    assert (((words[:, None] >> np.arange(32, dtype=np.uint32)[None, :]) & 1).reshape(-1)[P:] == 0).all()
    c = int(count.item())
    assert c == want.size
    np.testing.assert_array_equal(idx.cpu().numpy()[:c], want)
    return want.size


@pytest.mark.parametrize("tau", [0, 1, 20, 45, 60, 100, 127])
def test_filter_c1_thresholds(tau):
    q, t = synth.gen_pairs(synth.seed_for_config(1), 1024, 64, 64, planted=True)
    _check_filter(q, t, tau, s=8)


@pytest.mark.parametrize("P,m,n,tau", [(1000, 40, 56, 30), (33, 128, 128, 100), (4096, 128, 128, 110),
                                       (300, 300, 300, 200), (257, 64, 1024, 70), (100, 9, 1, 1)])
def test_filter_shapes(P, m, n, tau):
    q, t = synth.gen_pairs(8080 + m + n, P, m, n, planted=True)
    _check_filter(q, t, tau)


@pytest.mark.parametrize("consts", [(1, -1, -1), (3, -2, -1), (1, 0, 0), (5, -3, -4)])
def test_filter_runtime_constants(consts):
    q, t = synth.gen_pairs(8181, 500, 37, 61, planted=True)
    c1, mm, g = consts
    for tau in (5, 20, 40):
        _check_filter(q, t, tau, c1, mm, g, 12)


def test_filter_threshold_edges():
    q, t = synth.gen_pairs(8282, 70, 20, 30, planted=True)
    assert _check_filter(q, t, 40) == 0  # >= match * min(m, n): nothing can exceed it
    dq = torch.from_numpy(q).to(DEV)
    dt = torch.from_numpy(t).to(DEV)
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.filter_batch(dq, dt, 255, score_bits=8)  # > 2^s - 2
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.filter_batch(dq, dt, -1, score_bits=8)
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG


# ---------------------------------------------------------------- wordwise comparator (NEXT-4)


@pytest.mark.parametrize("P,m,n", [(1, 1, 1), (33, 9, 5), (1000, 40, 56), (4096, 128, 128),
                                   (777, 256, 300), (500, 64, 1024), (301, 200, 90), (64, 32, 32)])
def test_wordwise_matches_oracle(P, m, n):
    q, t = synth.gen_pairs(9191 + m + n, P, m, n, planted=True)
    dq = torch.from_numpy(q).to(DEV)
    dt = torch.from_numpy(t).to(DEV)
    got = bpbc.score_batch_wordwise(dq, dt, 2, -1, -1).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1))


@pytest.mark.parametrize("consts", [(1, -1, -1), (3, -2, -1), (1, 0, 0), (5, -3, -4), (2, -7, -1)])
def test_wordwise_runtime_constants(consts):
    q, t = synth.gen_pairs(9292, 300, 37, 61, planted=True)
    c1, mm, g = consts
    got = bpbc.score_batch_wordwise(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                                    c1, mm, g).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, c1, mm, g))


def test_wordwise_agrees_with_bitwise_at_c2_size():
    """The two independent GPU algorithms agree on a full C2-sized batch."""
    q, t = synth.gen_pairs(synth.seed_for_config(2), 1 << 20, 128, 128)
    dq = torch.from_numpy(q).to(DEV)
    dt = torch.from_numpy(t).to(DEV)
    a = bpbc.score_batch_wordwise(dq, dt, 2, -1, -1)
    b = bpbc.score_batch(dq, dt, 2, -1, -1, score_bits=9)
    assert torch.equal(a, b)


def test_c5_point_full_size_sampled():
    """BASELINE config 5's largest point at full size: 2^22 pairs, m = n = 512,
    11-bit slices (the multi-warp kernel), checked on a seeded sample."""
    _sampled(5, 1 << 22, 512, 512, 11, sample=512)
    assert bpbc.last_plan(0)["lanes"] == 128  # 4 warps x 32 lanes per group


def test_filter_c2_full_size_sampled():
    """Threshold filter at C2's size: the flagged set on a sample equals the
    oracle's, and the count equals the number of set mask bits."""
    P, m, n, tau = 1 << 20, 128, 128, 110
    q, t = synth.gen_pairs(synth.seed_for_config(2), P, m, n, planted=True)
    mask, count, idx = bpbc.filter_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                                         tau, score_bits=9)
    words = mask.cpu().numpy().view(np.uint32)
    bits = ((words[:, None] >> np.arange(32, dtype=np.uint32)[None, :]) & 1).reshape(-1)
    c = int(count.item())
    assert c == int(bits.sum())
    got_idx = idx.cpu().numpy()[:c]
    assert np.all(np.diff(got_idx) > 0)
    np.testing.assert_array_equal(got_idx, np.nonzero(bits)[0])
    rng = np.random.default_rng(2)
    sample = np.sort(rng.choice(P, size=4096, replace=False))
    want = oracle.sw_batch(q[sample], t[sample], 2, -1, -1) > tau
    np.testing.assert_array_equal(bits[sample].astype(bool), want)


# ---------------------------------------------------------------- few long groups (row-skewed kernel)


@pytest.mark.parametrize("P,m,n", [(2048, 128, 4096), (100, 100, 4000), (64, 97, 3200), (33, 128, 5000)])
def test_few_long_groups(P, m, n):
    """Few groups of long targets (the paper's shape, scaled down), incl.
    padded rows, ragged n (chunks straddling groups) and ragged P."""
    q, t = synth.gen_pairs(5150 + m + n, P, m, n, planted=True)
    check_full(q, t)


def test_few_long_groups_constants_and_filter():
    q, t = synth.gen_pairs(5252, 96, 120, 3900, planted=True)
    check_full(q, t, 3, -2, -1, 12)
    _check_filter(q, t, 150)


@pytest.mark.parametrize("m,n", [(64, 64), (128, 200), (300, 300)])
def test_bad_base_flag_all_kernels(m, n):
    """Codes > 3 are read as c & 3 and raise the sticky flag in the fused
    sweep (transposes raw codes itself), the multi-warp path (pack kernel)."""
    q, t = synth.gen_pairs(99 + m, 64, m, n)
    bpbc.get_error_flags(0)  # clear
    t2 = t.copy()
    t2[7, n - 1] = 0xFF
    got = run(q, t2)
    assert bpbc.get_error_flags(0) & _lib.BPBC_FLAG_BAD_BASE
    np.testing.assert_array_equal(
        got, oracle.sw_batch(q, t2 & 3, 2, -1, -1, score_bits=bpbc.default_score_bits(2, m, n)))
    run(q, t)
    assert bpbc.get_error_flags(0) == 0


def _sharded_worker(rank, world, port, P, m, n, path):
    import os
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_nishimurabin17_b200 import parallel
        b, e = parallel.shard_range(P, world, rank)
        q, t = synth.gen_pairs(4545, e - b, m, n, planted=True, p_offset=b)
        local = parallel.score_sharded(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV), P,
                                       2, -1, -1, 9)
        full = parallel.gather_scores(local.cpu(), P)  # gloo gathers host tensors
        if rank == 0:
            np.save(path, full.numpy())
    finally:
        dist.destroy_process_group()


def test_score_sharded_two_ranks_one_gpu(tmp_path):
    """parallel.score_sharded under torch.distributed: 2 ranks (sharing cuda:0,
    gloo for the gather) score their shards; the gathered scores equal the
    oracle's for the whole batch."""
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    P, m, n = 3000, 96, 128
    path = str(tmp_path / "sharded.npy")
    mp.spawn(_sharded_worker, args=(2, port, P, m, n, path), nprocs=2, join=True)
    q, t = synth.gen_pairs(4545, P, m, n, planted=True)
    np.testing.assert_array_equal(np.load(path), oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))
