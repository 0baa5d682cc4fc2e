"""GPU parity of the wrap-around schedule and the paper's own
workload (32768 pairs, m = 128, n = 1024 ... 65536).

The wrap-around schedule splits groups between streams and hands the split
group's whole warp state over as a snapshot; every test here compares the
result with the CPU oracle element by element (bit-exact), and checks that
the plan actually used the schedule under test.
"""
import os
import threading

import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_ipps_nishimurabin17_b200 as bpbc

pytestmark = pytest.mark.gpu

DEV = "cuda:0"


def in_thread_with_env(env, fn):
    """Run fn() in a new host thread (so it gets its own ctx, which reads the
    environment at bpbc_sw_init) with extra environment variables set."""
    box = {}
    old = {k: os.environ.get(k) for k in env}

    def run():
        try:
            box["out"] = fn()
        except BaseException as exc:  # re-raised in the caller
            box["exc"] = exc
        finally:
            bpbc.release_thread_ctx(0)

    os.environ.update(env)
    try:
        th = threading.Thread(target=run)
        th.start()
        th.join()
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
    if "exc" in box:
        raise box["exc"]
    return box["out"]


def gpu_scores(q, t, match=2, mismatch=-1, gap=-1, s=None):
    dq = torch.from_numpy(np.ascontiguousarray(q)).to(DEV)
    dt = torch.from_numpy(np.ascontiguousarray(t)).to(DEV)
    out = bpbc.score_batch(dq, dt, match, mismatch, gap, score_bits=s).cpu().numpy()
    return out, bpbc.last_plan(0)


def check(q, t, match=2, mismatch=-1, gap=-1, s=None, expect_wrap=True):
    m, n = q.shape[1], t.shape[1]
    if s is None:
        s = bpbc.default_score_bits(match, m, n)
    got, plan = gpu_scores(q, t, match, mismatch, gap, s)
    if expect_wrap is not None:
        assert plan["wrap"] == expect_wrap, plan
    want = oracle.sw_batch(q, t, match, mismatch, gap, score_bits=s)
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, (f"{bad.size}/{len(want)} mismatches (m={m} n={n} s={s} plan={plan}); "
                           f"first pair {bad[0]}: got {got[bad[0]]} want {want[bad[0]]}")
    return got, plan


# ---------------------------------------------------------------- wrap-around schedule


@pytest.mark.parametrize("groups,m,n", [(700, 128, 1024), (600, 128, 2048), (600, 100, 2048),
                                        (1024, 128, 1536), (640, 200, 1024), (620, 256, 512)])
def test_wrap_schedule_matches_oracle(groups, m, n):
    """Few groups of long targets: the planner picks the wrap-around schedule
    (R = 4 and R = 8 tilings, padded rows) and the scores are exact."""
    q, t = synth.gen_pairs(7300 + groups + m + n, groups * 32, m, n, planted=True)
    check(q, t)


def test_wrap_ragged_pairs_and_packed2():
    """A ragged last group (P % 32 != 0) and 2-bit packed input under the
    wrap-around schedule."""
    P, m, n = 650 * 32 - 7, 128, 1024
    q, t = synth.gen_pairs(7401, P, m, n, planted=True)
    check(q, t)
    q2 = torch.from_numpy(synth.pack2bit(q)).to(DEV)
    t2 = torch.from_numpy(synth.pack2bit(t)).to(DEV)
    got = bpbc.score_batch_packed2(q2, t2, m, n, 2, -1, -1).cpu().numpy()
    assert bpbc.last_plan(0)["wrap"]
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))


@pytest.mark.parametrize("consts,s", [((3, -2, -2), 12), ((1, -1, -1), 10), ((1, -3, -5), 12),
                                      ((2, 0, -1), 9), ((5, -4, -4), 12)])
def test_wrap_runtime_constants(consts, s):
    """Runtime constants: the exact circuit with masks (g >= c2) and the
    saturating circuit (g < c2) under the wrap-around schedule."""
    q, t = synth.gen_pairs(7500 + s, 600 * 32, 96, 1024, planted=True)
    check(q, t, *consts, s=s)


def test_wrap_saturating_width():
    """Width below s_exact: the saturating circuit saturates planted pairs;
    out = min(exact, 2^s - 1) (R3) under the wrap-around schedule."""
    q, t = synth.gen_pairs(7600, 600 * 32, 128, 1024, planted=True)
    got, _ = check(q, t, s=7)
    assert (got == 127).any()


def test_wrap_filter():
    """Threshold filter (NEXT-2) under the wrap-around schedule: the flag word
    travels in the snapshot."""
    P, m, n, tau = 600 * 32, 128, 1024, 110
    q, t = synth.gen_pairs(7700, P, m, n, planted=True)
    mask, count, idx = bpbc.filter_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                                         tau, score_bits=9)
    want = np.nonzero(oracle.sw_batch(q, t, 2, -1, -1) > tau)[0]
    c = int(count.item())
    assert c == want.size and c > 0
    np.testing.assert_array_equal(idx.cpu().numpy()[:c], want)


def test_wrap_forced_equals_group_granular():
    """The same batch through the forced wrap-around schedule (BPBC_WRAP=1)
    and the forced group-granular split (BPBC_WRAP=0) gives identical scores,
    equal to the oracle's, for a shape the planner would not wrap."""
    P, m, n = 1200 * 32, 128, 512
    q, t = synth.gen_pairs(7800, P, m, n, planted=True)
    want = oracle.sw_batch(q, t, 2, -1, -1, score_bits=9)
    a, pa = in_thread_with_env({"BPBC_WRAP": "1"}, lambda: gpu_scores(q, t, s=9))
    b, pb = in_thread_with_env({"BPBC_WRAP": "0"}, lambda: gpu_scores(q, t, s=9))
    assert pa["wrap"] and not pb["wrap"]
    np.testing.assert_array_equal(a, want)
    np.testing.assert_array_equal(b, want)


@pytest.mark.parametrize("blocks", ["1", "2", "3"])
def test_wrap_blocks_per_sm(blocks):
    """Forced wrap at 1..3 resident blocks per SM (more streams, shorter
    spans, more snapshot hand-offs per group)."""
    P, m, n = 2400 * 32, 128, 1024
    q, t = synth.gen_pairs(7900 + int(blocks), P, m, n, planted=True)
    got, plan = in_thread_with_env({"BPBC_WRAP": "1", "BPBC_MAX_BLOCKS_PER_SM": blocks},
                                   lambda: gpu_scores(q, t, s=9))
    assert plan["wrap"] and plan["blocks_per_sm"] <= int(blocks)
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))


# ---------------------------------------------------------------- the paper's shape (NEXT-3)

PAPER_P, PAPER_M = 32768, 128


@pytest.mark.parametrize("n", [1024, 8192])
def test_paper_shape_full_parity(n):
    """The paper's workload (32768 pairs, m = 128) at n = 1024 and
    8192, every pair checked against the oracle, in the launch configuration
    bench.py times (the planner's wrap-around schedule)."""
    q, t = synth.gen_pairs(synth.seed_for_config(6) + n, PAPER_P, PAPER_M, n, planted=True)
    check(q, t, s=9)


def test_paper_shape_n65536_sampled():
    """n = 65536 (the paper's longest target, 2.7e11 cells): 4096 sampled
    pairs (and the first and last) against the oracle; every score within
    [0, min(2 m, 2^s - 1)]."""
    n = 65536
    q, t = synth.gen_pairs(synth.seed_for_config(6), PAPER_P, PAPER_M, n, planted=True)
    got, plan = gpu_scores(q, t, s=9)
    assert plan["wrap"], plan
    rng = np.random.default_rng(65536)
    idx = np.sort(np.concatenate([rng.choice(PAPER_P, size=4096, replace=False), [0, PAPER_P - 1]]))
    np.testing.assert_array_equal(got[idx], oracle.sw_batch(q[idx], t[idx], 2, -1, -1,
                                                            score_bits=9))
    assert got.min() >= 0 and got.max() <= 2 * PAPER_M
