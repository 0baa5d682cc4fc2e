"""Pins of the CPU oracle against values fixed by the paper and by mathematics.

Every function in oracle/ is checked here against something other than
itself: the paper's worked examples (tests/golden/, with citations), brute
force enumeration, textbook special cases (LCS, longest common substring,
Kadane), closed forms and invariants.  CPU only.
"""
import itertools
import os
import random

import numpy as np
import pytest

import oracle
import synth
from tests import pins

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

CONSTS = [(2, -1, -1), (1, -1, -1), (3, -2, -1), (1, 0, 0), (2, -3, -2), (5, -1, -4),
          (1, -1, 0), (2, 0, -1)]


def _read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


# --------------------------------------------------------------------------
# Paper worked examples


def test_table2_matrix_cell_by_cell():
    """Table II: all 48 cells and the max 8."""
    rows = _read_golden("table2.txt")
    kv = {r[0]: r[1] for r in rows if len(r) == 2}
    mat = np.array([[int(v) for v in r] for r in rows if len(r) > 2], dtype=np.int32)
    x, y = synth.encode(kv["X"]), synth.encode(kv["Y"])
    args = (int(kv["match"]), int(kv["mismatch"]), int(kv["gap"]))
    d = oracle.sw_matrix(x, y, *args)
    assert d.shape == (6, 8)
    np.testing.assert_array_equal(d, mat)
    assert oracle.sw_score(x, y, *args) == 8
    # the max is at (x_5, y_6) (1-based), the alignment ACTG/ACTG of P:L218
    assert np.unravel_index(np.argmax(d), d.shape) == (5, 6)


def test_table2_rules_out_literal_gap_sign():
    """Reading R1: subtracting the printed gap = -1 literally (i.e. adding 1)
    does not reproduce Table II (max would be 11, not 8)."""
    x, y = synth.encode("TACTG"), synth.encode("GAACTGA")
    assert oracle.sw_score(x, y, 2, -1, +1) == 11
    assert oracle.sw_score(x, y, 2, -1, -1) == 8


def test_table3_wavefront_times():
    """Table III prints 1-based t for the cells; reading R7: the
    0-based wavefront index of cell (i, j) is t = i + j."""
    table3 = [[1, 2, 3, 4, 5, 6, 7], [2, 3, 4, 5, 6, 7, 8], [3, 4, 5, 6, 7, 8, 9],
              [4, 5, 6, 7, 8, 9, 10], [5, 6, 7, 8, 9, 10, 11]]
    for i in range(5):
        for j in range(7):
            assert table3[i][j] == i + j + 1


def test_sec2_bit_transpose_example():
    """the bit-transpose planes of the 4-pair example, bit k = pair k."""
    rows = _read_golden("sec2_planes.txt")
    pairs = [r for r in rows if r[0].startswith("X") and len(r) == 4]
    xs = [synth.encode(r[1]) for r in pairs]
    ys = [synth.encode(r[3]) for r in pairs]
    planes_x = oracle.pack_planes(np.stack(xs))
    planes_y = oracle.pack_planes(np.stack(ys))
    kv = {r[0]: r[1:] for r in rows}
    for i, w in enumerate(kv["XH"]):
        assert planes_x[0, i, 0] == pins.bits_to_word(w)
    for i, w in enumerate(kv["XL"]):
        assert planes_x[0, i, 1] == pins.bits_to_word(w)
    for j, w in enumerate(kv["YH"]):
        assert planes_y[0, j, 0] == pins.bits_to_word(w)
    for j, w in enumerate(kv["YL"]):
        assert planes_y[0, j, 1] == pins.bits_to_word(w)
    # BPBC straightforward string matching on these planes gives the
    # bitwise complement of the printed d (reading R11).
    m, n = 5, 8
    for j, printed in enumerate(kv["d"]):
        d = 0
        for i in range(m):
            d |= int(planes_x[0, i, 0] ^ planes_y[0, i + j, 0]) | int(
                planes_x[0, i, 1] ^ planes_y[0, i + j, 1])
        assert d & 0xF == (~pins.bits_to_word(printed)) & 0xF


def test_sec2_single_pair_match_string():
    """X=ATTCG in Y=AAATTCGGGA gives d = 110111 (0 = occurrence)."""
    x, y = synth.encode("ATTCG"), synth.encode("AAATTCGGGA")
    planes_x = oracle.pack_planes(x[None, :])
    planes_y = oracle.pack_planes(y[None, :])
    bits = ""
    for j in range(len(y) - len(x) + 1):
        d = 0
        for i in range(len(x)):
            d |= int(planes_x[0, i, 0] ^ planes_y[0, i + j, 0]) | int(
                planes_x[0, i, 1] ^ planes_y[0, i + j, 1])
        bits += str(d & 1)
    assert bits == "110111"


# --------------------------------------------------------------------------
# Brute force


@pytest.mark.parametrize("consts", CONSTS)
def test_brute_force_exhaustive_small(consts):
    """Every pair with 1 <= m, n <= 3 (4^(m+n) pairs each): DP == enumeration."""
    for m in range(1, 4):
        for n in range(1, 4):
            for xs in itertools.product(range(4), repeat=m):
                for ys in itertools.product(range(4), repeat=n):
                    a = oracle.sw_score(xs, ys, *consts)
                    b = oracle.brute_local(xs, ys, *consts)
                    assert a == b, (xs, ys, consts, a, b)


def test_brute_force_random():
    rng = random.Random(1234)
    for _ in range(400):
        m, n = rng.randint(1, 7), rng.randint(1, 7)
        xs = [rng.randrange(4) for _ in range(m)]
        ys = [rng.randrange(4) for _ in range(n)]
        c = (rng.randint(1, 6), -rng.randint(0, 6), -rng.randint(0, 6))
        assert oracle.sw_score(xs, ys, *c) == oracle.brute_local(xs, ys, *c)


# --------------------------------------------------------------------------
# Special cases that reduce to textbook routines


def test_gap_zero_is_match_times_lcs():
    rng = random.Random(7)
    for _ in range(300):
        m, n = rng.randint(1, 16), rng.randint(1, 16)
        xs = [rng.randrange(4) for _ in range(m)]
        ys = [rng.randrange(4) for _ in range(n)]
        match, mismatch = rng.randint(1, 5), -rng.randint(0, 5)
        assert oracle.sw_score(xs, ys, match, mismatch, 0) == match * pins.lcs_len(xs, ys)


def test_huge_penalties_is_longest_common_substring():
    rng = random.Random(8)
    for _ in range(300):
        m, n = rng.randint(1, 16), rng.randint(1, 16)
        xs = [rng.randrange(4) for _ in range(m)]
        ys = [rng.randrange(4) for _ in range(n)]
        match = rng.randint(1, 5)
        big = -(match * min(m, n) + 1)
        assert oracle.sw_score(xs, ys, match, big, big) == \
            match * pins.longest_common_substring(xs, ys)


def test_huge_gap_is_diagonal_kadane():
    rng = random.Random(9)
    for _ in range(300):
        m, n = rng.randint(1, 16), rng.randint(1, 16)
        xs = [rng.randrange(4) for _ in range(m)]
        ys = [rng.randrange(4) for _ in range(n)]
        match, mismatch = rng.randint(1, 5), -rng.randint(0, 5)
        big = -(match * min(m, n) + 1)
        assert oracle.sw_score(xs, ys, match, mismatch, big) == \
            pins.best_diagonal_kadane(xs, ys, match, mismatch)


# --------------------------------------------------------------------------
# Closed forms


def test_closed_forms():
    rng = random.Random(10)
    for _ in range(100):
        m = rng.randint(1, 64)
        xs = [rng.randrange(4) for _ in range(m)]
        c = (rng.randint(1, 5), -rng.randint(0, 5), -rng.randint(0, 5))
        assert oracle.sw_score(xs, xs, *c) == m * c[0]                    # X = Y
        n = rng.randint(1, 64)
        assert oracle.sw_score([0] * m, [0] * n, *c) == c[0] * min(m, n)  # A^m vs A^n
        # disjoint base sets {A,T} vs {G,C}: no positive alignment
        ys = [rng.choice([2, 3]) for _ in range(n)]
        xa = [rng.choice([0, 1]) for _ in range(m)]
        assert oracle.sw_score(xa, ys, *c) == 0


# --------------------------------------------------------------------------
# Invariants on seeded batches


def test_invariants_batch():
    P, m, n = 512, 24, 40
    q, t = synth.gen_pairs(synth.seed_for_config(99), P, m, n, planted=True)
    for c in [(2, -1, -1), (3, -2, -2), (1, 0, -1)]:
        base = oracle.sw_batch(q, t, *c)
        assert (base >= 0).all() and (base <= c[0] * min(m, n)).all()
        # per-pair == batch
        for p in range(0, P, 37):
            assert base[p] == oracle.sw_score(q[p], t[p], *c)
        # symmetry under swapping query and target
        np.testing.assert_array_equal(oracle.sw_batch(t, q, *c), base)
        # reversal of both sequences
        np.testing.assert_array_equal(oracle.sw_batch(q[:, ::-1], t[:, ::-1], *c), base)
        # base relabelling (any permutation applied to both)
        for perm in ([3, 2, 1, 0], [1, 0, 3, 2], [2, 3, 0, 1], [0, 2, 1, 3]):
            pm = np.array(perm, dtype=np.uint8)
            np.testing.assert_array_equal(oracle.sw_batch(pm[q], pm[t], *c), base)
        # monotone under appending characters
        q2, t2 = synth.gen_pairs(7, P, 3, 5)
        ext = oracle.sw_batch(np.concatenate([q, q2], 1), np.concatenate([t, t2], 1), *c)
        assert (ext >= base).all()
        # thread count does not matter
        np.testing.assert_array_equal(oracle.sw_batch(q, t, *c, threads=1), base)


def test_width_cap_law():
    """out(s) = min(exact, 2^s - 1) (reading R3) and the cross-width law."""
    P, m, n = 256, 64, 64
    q, t = synth.gen_pairs(synth.seed_for_config(1), P, m, n, planted=True)
    exact = oracle.sw_batch(q, t, 2, -1, -1)
    assert exact.max() == 128  # planted exact copies reach m * match
    for s in range(4, 10):
        capped = oracle.sw_batch(q, t, 2, -1, -1, score_bits=s)
        np.testing.assert_array_equal(capped, np.minimum(exact, 2 ** s - 1))
        for s2 in range(s, 10):
            np.testing.assert_array_equal(
                capped, np.minimum(oracle.sw_batch(q, t, 2, -1, -1, score_bits=s2), 2 ** s - 1))


def test_exact_width_fits():
    """Reading R2: s = bit_length(match * min(m, n)) never saturates; one bit
    less saturates the self-alignment."""
    for m in [32, 64, 128, 256]:
        x = np.array([i % 4 for i in range(m)], dtype=np.uint8)[None, :]
        s = (2 * m).bit_length()
        assert oracle.sw_batch(x, x, 2, -1, -1, score_bits=s)[0] == 2 * m
        assert oracle.sw_batch(x, x, 2, -1, -1, score_bits=s - 1)[0] == 2 ** (s - 1) - 1


# --------------------------------------------------------------------------
# pack / untranspose definitions


def test_untranspose_definition():
    rng = np.random.default_rng(3)
    for s in [4, 9, 16]:
        vals = rng.integers(0, 2 ** s, size=64)
        planes = np.stack([pins.planes_from_scores(vals[:32], s),
                           pins.planes_from_scores(vals[32:], s)])
        np.testing.assert_array_equal(oracle.untranspose(planes), vals)


def test_pack_roundtrip_and_padding():
    rng = np.random.default_rng(4)
    codes = rng.integers(0, 4, size=(45, 13), dtype=np.uint8)
    planes = oracle.pack_planes(codes)
    assert planes.shape == (2, 13, 2)
    for i in range(13):
        # planes [H, L] -> 2-bit value per pair = 2H + L
        two = np.stack([planes[:, i, 1], planes[:, i, 0]], axis=1)  # bit0 = L, bit1 = H
        got = oracle.untranspose(two)[:45]
        np.testing.assert_array_equal(got, codes[:, i])
    # pairs 45..63 are padding: code 0
    assert (planes[1] >> np.uint32(13) == 0).all()


def test_generator_c_matches_numpy_definition():
    for planted in (False, True):
        for (P, m, n, off) in [(300, 7, 11, 0), (130, 64, 64, 12345), (65, 1, 3, 2 ** 30)]:
            a = synth.gen_pairs(77, P, m, n, planted=planted, p_offset=off)
            b = synth.gen_pairs_np(77, P, m, n, planted=planted, p_offset=off)
            np.testing.assert_array_equal(a[0], b[0])
            np.testing.assert_array_equal(a[1], b[1])
    q, _ = synth.gen_pairs(1, 4096, 64, 1)
    frac = np.bincount(q.ravel(), minlength=4) / q.size
    assert np.all(np.abs(frac - 0.25) < 0.01)


def test_pack2bit_roundtrip_and_layout():
    """Input-format helper of the packed2 entry points: base i in bits 2(i%4)
    of byte i//4 (include/bpbc_sw.h), lossless for codes 0..3."""
    rng = np.random.default_rng(5)
    for ln in (1, 3, 4, 5, 31, 64, 129):
        c = rng.integers(0, 4, size=(7, ln), dtype=np.uint8)
        p = synth.pack2bit(c)
        assert p.shape == (7, (ln + 3) // 4)
        np.testing.assert_array_equal(synth.unpack2bit(p, ln), c)
    # hand example: ATGC -> 0 | 1<<2 | 2<<4 | 3<<6 = 0b11100100
    assert synth.pack2bit(synth.encode("ATGC")[None, :])[0, 0] == 0b11100100
