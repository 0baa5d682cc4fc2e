"""SASS regression pins of the headline sweep kernels (no GPU needed): the
switch-free hot loop of each kernel issues the circuit's hand-counted LOP3
per word-cell (10 S for the exact circuit, 11 S + 2 for the
saturating one; the paper's count is Theorem 6), carries no local-
memory traffic, and adds at most ~7 % other instructions.  The committed
table is profiles/r2_sass_loops.md (tools/sass_report.py).
"""
import os
import shutil
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

pytestmark = pytest.mark.skipif(shutil.which("cuobjdump") is None or shutil.which("nm") is None,
                                reason="no cuobjdump / nm")
BUILD = os.path.join(ROOT, "build", "csrc")


@pytest.fixture(scope="module")
def rows():
    if not os.path.exists(os.path.join(BUILD, "sweep_s9_m0.o")):
        pytest.skip("build/csrc objects not built")
    import sass_report
    return sass_report.report(BUILD)


def test_every_headline_kernel_found(rows):
    assert all("error" not in r for r in rows), [r for r in rows if "error" in r]


def test_lop3_per_word_cell_matches_hand_count(rows):
    for r in rows:
        assert abs(r["lop3_per_word_cell"] - r["hand_count"]) <= 0.02 * r["hand_count"], r["kernel"]


def test_exact_circuit_loops_are_exactly_10s(rows):
    """The switch-free loops of the exact (+2,-1,-1) single-warp kernels:
    LOP3 per word-cell equals 10 S exactly (C1/C4, C2, m=32, paper shape)."""
    for r in rows:
        if r["kernel"].startswith(("C1/C4", "C2 (", "C5 m=32", "paper shape")):
            assert r["lop3_per_word_cell"] == r["hand_count"], r["kernel"]
            assert r["instructions"] <= 1.13 * r["lop3"], (r["kernel"], r["other"])


def test_hot_loops_do_not_touch_local_memory(rows):
    for r in rows:
        assert "LDL" not in r["other"] and "STL" not in r["other"], r["kernel"]
