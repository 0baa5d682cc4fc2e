"""Resource checks of the built sm_100a kernels (no GPU needed): the sweep
kernels the plans pick for BASELINE.json's configs use no local memory
(no register spills) and fit the register budget that gives their planned
occupancy.  Reads `cuobjdump -res-usage` of the library.
"""
import re
import shutil
import subprocess

import pytest

from paper_conf_ipps_nishimurabin17_b200 import _lib

pytestmark = pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="no cuobjdump")


@pytest.fixture(scope="module")
def usage():
    out = subprocess.run(["cuobjdump", "-res-usage", _lib.LIB_PATH], capture_output=True,
                         text=True).stdout
    res = {}
    name = None
    for ln in out.splitlines():
        m = re.match(r"\s*Function (\S+):", ln)
        if m:
            name = m.group(1)
            continue
        m = re.search(r"REG:(\d+) STACK:(\d+) SHARED:(\d+) LOCAL:(\d+)", ln)
        if m and name:
            res.setdefault(name, []).append(tuple(int(x) for x in m.groups()))
    assert res, "no kernels found"
    return res


def find(usage, pattern):
    hits = [v for k, vs in usage.items() if re.search(pattern, k) for v in vs]
    assert hits, pattern
    return hits


# (kernel symbol pattern, max registers) for the plans of C1..C5 (+2/-1/-1)
HEADLINE = [
    (r"sw_sweep_kernelILi8ELi4ELi16ELi0ELb0ENS_4KFixILi2ELi1ELi1EEELb0E", 128),   # C1, C4 (s=8, 64 rows)
    (r"sw_sweep_kernelILi9ELi4ELi32ELi0ELb0ENS_4KFixILi2ELi1ELi1EEELb0E", 128),   # C2 (s=9, 128 rows)
    (r"sw_sweep_kernelILi10ELi8ELi32ELi0ELb0ENS_4KFixILi2ELi1ELi1EEELb0E", 255),  # C3 (s=10, 256 rows)
    (r"sw_sweep_mw_kernelILi11ELi4ELi4ELi0ENS_4KFixILi2ELi1ELi1E", 168),    # C5 point (512 rows)
]


@pytest.mark.parametrize("pattern,max_regs", HEADLINE)
def test_headline_kernels_do_not_spill(usage, pattern, max_regs):
    # Each pattern matches the max-mode and the threshold-mode instantiation.
    # ptxas keeps up to 16 bytes of cold state (group-switch path) on the
    # stack in a few of them (C5's multi-warp kernel at its forced 128
    # registers; the C4 threshold variant); anything larger is a real spill.
    for reg, stack, shared, local in find(usage, pattern):
        assert local == 0 and stack <= 16, (pattern, reg, stack, local)
        assert reg <= max_regs, (pattern, reg)


def test_host_streamed_variants_do_not_spill(usage):
    """The host-streamed (polling) instantiations of the headline fused
    kernels (HS = true, the host-buffer path only) may take more registers
    (the C1/C4 one: ~150, 3 blocks/SM) but never spill."""
    for pattern, _ in HEADLINE[:3]:
        for reg, stack, shared, local in find(usage, pattern[:-2] + "1E"):
            assert local == 0 and stack <= 16, (pattern, reg, stack, local)


def test_c2_kernel_has_no_stack_at_all(usage):
    """The headline C2 sweep (both modes): no stack frame, <= 128 registers."""
    for reg, stack, shared, local in find(usage, HEADLINE[1][0]):
        assert stack == 0 and local == 0 and reg <= 128, (reg, stack)


def test_pack_and_extract_do_not_spill(usage):
    for pat in (r"pack_kernel", r"extract_kernel", r"filter_mask_kernel", r"wordwise_kernel"):
        for reg, stack, shared, local in find(usage, pat):
            assert local == 0, (pat, reg, local)
