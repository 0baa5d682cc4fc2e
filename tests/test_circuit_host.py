"""Host checks of the product's bit-sliced cell circuits (csrc/circuit.cuh).

The same header the CUDA kernels include is compiled for the host (lop3
emulated) by tests/circuit_harness.cpp and checked:
  * exhaustively against integer arithmetic for every (up, left, diag, e) at
    small widths, for the exact and the saturating cells;
  * end to end: a row-major bit-sliced DP of 32-pair groups with these
    circuits equals min(oracle score, 2^s - 1) (reading R3), including
    planted pairs that hit the cap.
CPU only.
"""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import oracle
import synth

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRC = os.path.join(HERE, "circuit_harness.cpp")
HDR = os.path.join(ROOT, "paper_conf_ipps_nishimurabin17_b200", "csrc", "circuit.cuh")
LIB = os.path.join(HERE, "_build", "libcircuit_harness.so")


@pytest.fixture(scope="module")
def harness():
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    if (not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(SRC),
                                                                 os.path.getmtime(HDR))):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-o", tmp, SRC])
        os.replace(tmp, LIB)
    lib = ctypes.CDLL(LIB)
    lib.harness_exhaustive.restype = ctypes.c_longlong
    lib.harness_exhaustive.argtypes = [ctypes.c_int] * 6
    lib.harness_group_dp.restype = ctypes.c_int
    lib.harness_group_dp.argtypes = [ctypes.c_int] * 5 + [ctypes.c_void_p, ctypes.c_int,
                                                          ctypes.c_void_p, ctypes.c_int,
                                                          ctypes.c_void_p]
    lib.harness_gate_tables.restype = ctypes.c_int
    return lib


def test_gate_tables(harness):
    assert harness.harness_gate_tables() == 0


@pytest.mark.parametrize("S", [4, 5, 6, 7])
@pytest.mark.parametrize("kill", [0, 1])
def test_exact_cell_exhaustive(harness, S, kill):
    assert harness.harness_exhaustive(0, S, 2, 1, 1, kill) == 0


@pytest.mark.parametrize("S", [4, 5, 6, 7])
def test_sat_cell_fixed_exhaustive(harness, S):
    assert harness.harness_exhaustive(1, S, 2, 1, 1, 0) == 0


@pytest.mark.parametrize("consts", [(2, 1, 1), (1, 1, 1), (3, 2, 1), (1, 0, 0), (5, 3, 4),
                                    (2, 0, 1), (1, 7, 0), (15, 15, 15)])
@pytest.mark.parametrize("S", [4, 5, 6])
def test_sat_cell_runtime_exhaustive(harness, S, consts):
    c1, c2, g = consts
    if max(consts) > 2 ** S - 1:
        pytest.skip("constants must fit in S bits")
    assert harness.harness_exhaustive(2, S, c1, c2, g, 0) == 0


@pytest.mark.parametrize("consts", [(2, 1, 1), (1, 1, 1), (3, 2, 2), (1, 3, 5), (1, 0, 0),
                                    (2, 0, 3), (4, 1, 2)])
@pytest.mark.parametrize("S", [4, 5, 6])
@pytest.mark.parametrize("kill", [0, 1])
def test_exact_cell_runtime_exhaustive(harness, S, consts, kill):
    """Exact circuit with runtime constants (per-bit masks), any g >= c2."""
    c1, c2, g = consts
    if c1 + g > 2 ** S - 1:
        pytest.skip("c1 + g must fit in S bits")
    assert harness.harness_exhaustive(3, S, c1, c2, g, kill) == 0


def _group_scores(harness, circuit, S, consts, q, t):
    """Run the harness DP on each 32-pair group of q/t, return untransposed scores."""
    P, m = q.shape
    n = t.shape[1]
    xp = oracle.pack_planes(q)  # [G][m][2] -- the definition, not the kernel
    yp = oracle.pack_planes(t)
    G = xp.shape[0]
    M = np.zeros((G, S), dtype=np.uint32)
    for g in range(G):
        xg = np.ascontiguousarray(xp[g])
        yg = np.ascontiguousarray(yp[g])
        mo = np.zeros(S, dtype=np.uint32)
        rc = harness.harness_group_dp(circuit, S, consts[0], consts[1], consts[2],
                                      xg.ctypes.data, m, yg.ctypes.data, n, mo.ctypes.data)
        assert rc == 0
        M[g] = mo
    return oracle.untranspose(M)[:P]


@pytest.mark.parametrize("m,n", [(1, 1), (5, 7), (16, 16), (24, 40), (40, 24)])
def test_group_dp_exact_matches_oracle(harness, m, n):
    q, t = synth.gen_pairs(1001 + m * 7 + n, 96, m, n, planted=True)
    S = (2 * min(m, n) + 1).bit_length()
    S = max(S, 4)
    got = _group_scores(harness, 0, S, (2, 1, 1), q, t)
    want = oracle.sw_batch(q, t, 2, -1, -1, score_bits=S)
    np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("S", [4, 5, 6, 8])
@pytest.mark.parametrize("consts", [(2, 1, 1), (3, 2, 1), (1, 0, 2), (2, 3, 0)])
def test_group_dp_saturating_law(harness, S, consts):
    """Saturating circuit: DP max == min(exact, 2^S - 1) even when most pairs
    saturate (reading R3)."""
    m, n = 32, 48
    q, t = synth.gen_pairs(2002 + S, 128, m, n, planted=True)
    c1, c2, g = consts
    if max(consts) > 2 ** S - 1:
        pytest.skip("constants must fit")
    want = oracle.sw_batch(q, t, c1, -c2, -g, score_bits=S)
    if S <= 5:
        assert (want == 2 ** S - 1).any()  # the cap is really exercised
    for circuit in ([1, 2] if consts == (2, 1, 1) else [2]):
        got = _group_scores(harness, circuit, S, consts, q, t)
        np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("consts", [(2, 1, 1), (1, 1, 1), (3, 2, 2), (1, 3, 5), (5, 3, 4)])
@pytest.mark.parametrize("m,n", [(5, 7), (24, 40), (40, 24)])
def test_group_dp_exact_runtime_matches_oracle(harness, consts, m, n):
    """Exact circuit with runtime constants at its width bit_length(c1 min(m, n) + g):
    the group DP's max (over D', minus g) equals the oracle's score."""
    c1, c2, g = consts
    q, t = synth.gen_pairs(3003 + m * 7 + n + c1, 96, m, n, planted=True)
    S = max(4, (c1 * min(m, n) + g).bit_length())
    got = _group_scores(harness, 3, S, consts, q, t)
    want = oracle.sw_batch(q, t, c1, -c2, -g, score_bits=S)
    np.testing.assert_array_equal(got, want)
