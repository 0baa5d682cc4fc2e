"""GPU tests of the C-ABI boundary's stream, workspace and flag semantics
(include/bpbc_sw.h conventions): ctx-owned buffers across
streams, plan-exact workspace sizes, the BAD_BASE status of
bpbc_sw_get_error_flags, and the three-stream host-buffer path.  Every score
is checked against the CPU oracle.
"""
import ctypes

import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_ipps_nishimurabin17_b200 as bpbc
from paper_conf_ipps_nishimurabin17_b200 import _lib, api

pytestmark = pytest.mark.gpu

DEV = "cuda:0"


def test_ctx_workspace_ordered_across_streams():
    """workspace=NULL on two streams from one thread (one ctx): the second
    call waits for the first call's use of the ctx buffers (no silent
    corruption); the second batch is larger, so the buffer also grows while
    the first call may still be running."""
    qa, ta = synth.gen_pairs(8801, 40000, 128, 128, planted=True)
    qb, tb = synth.gen_pairs(8802, 70000, 128, 160, planted=True)
    da = [torch.from_numpy(x).to(DEV) for x in (qa, ta)]
    db = [torch.from_numpy(x).to(DEV) for x in (qb, tb)]
    s1, s2 = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    for _ in range(3):
        with torch.cuda.stream(s1):
            oa = bpbc.score_batch(*da, score_bits=9, stream=s1)
        with torch.cuda.stream(s2):
            ob = bpbc.score_batch(*db, score_bits=9, stream=s2)
        with torch.cuda.stream(s1):  # and back to the first stream
            oa2 = bpbc.score_batch(*db, score_bits=9, stream=s1)
    torch.cuda.synchronize()
    want_b = oracle.sw_batch(qb, tb, 2, -1, -1, score_bits=9)
    np.testing.assert_array_equal(oa.cpu().numpy(), oracle.sw_batch(qa, ta, 2, -1, -1, score_bits=9))
    np.testing.assert_array_equal(ob.cpu().numpy(), want_b)
    np.testing.assert_array_equal(oa2.cpu().numpy(), want_b)


@pytest.mark.parametrize("P,m,n,consts,s", [(5000, 128, 128, (2, -1, -1), 9),
                                            (3000, 300, 310, (2, -1, -1), 11),
                                            (2000, 700, 800, (1, -1, -1), 12),
                                            (20000, 128, 1024, (2, -1, -1), 9),
                                            (777, 40, 36, (3, -2, -1), 10)])
def test_workspace_bytes_for_is_exact(P, m, n, consts, s):
    """bpbc_sw_workspace_bytes_for gives the call's exact need: a caller
    workspace of exactly that size works, one byte less is INVALID_ARG, and
    it is never above the plan-free bound bpbc_sw_workspace_bytes."""
    q, t = synth.gen_pairs(8900 + m, P, m, n, planted=True)
    need = api.workspace_bytes_for(P, m, n, *consts, score_bits=s)
    assert 0 < need <= api.workspace_bytes(P, m, n)
    dq, dt = torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV)
    ws = torch.empty(need, dtype=torch.uint8, device=DEV)
    got = bpbc.score_batch(dq, dt, *consts, score_bits=s, workspace=ws).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, *consts, score_bits=s))
    with pytest.raises(bpbc.BPBCError) as ei:
        bpbc.score_batch(dq, dt, *consts, score_bits=s, workspace=ws[:need - 1])
    assert ei.value.status == _lib.BPBC_ERR_INVALID_ARG
    # the filter's compaction scratch lives in the workspace too
    fneed = api.workspace_bytes_for(P, m, n, *consts, score_bits=s, filter=True)
    assert need <= fneed <= api.workspace_bytes(P, m, n)
    fws = torch.empty(fneed, dtype=torch.uint8, device=DEV)
    tau = min(2 ** s - 2, 40)
    mask, count, idx = bpbc.filter_batch(dq, dt, tau, *consts, score_bits=s, workspace=fws)
    want = np.nonzero(oracle.sw_batch(q, t, *consts) > tau)[0]
    c = int(count.item())
    assert c == want.size
    np.testing.assert_array_equal(idx.cpu().numpy()[:c], want)


def test_get_error_flags_returns_bad_base_status():
    """The C call returns BPBC_ERR_BAD_BASE (and still writes and clears the
    flags) after a batch with a code > 3; BPBC_OK otherwise."""
    q, t = synth.gen_pairs(9001, 64, 30, 40)
    bpbc.get_error_flags(0)
    q2 = q.copy()
    q2[3, 7] = 9
    got = bpbc.score_batch(torch.from_numpy(q2).to(DEV), torch.from_numpy(t).to(DEV),
                           score_bits=8).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.sw_batch(q2 & 3, t, 2, -1, -1, score_bits=8))
    lib, ctx = _lib.load(), api._ctx(0)
    v = ctypes.c_uint32(0)
    assert lib.bpbc_sw_get_error_flags(ctx, ctypes.byref(v)) == _lib.BPBC_ERR_BAD_BASE
    assert v.value & _lib.BPBC_FLAG_BAD_BASE
    assert lib.bpbc_sw_get_error_flags(ctx, ctypes.byref(v)) == _lib.BPBC_OK and v.value == 0
    with pytest.raises(bpbc.BPBCError):
        bpbc.score_batch(torch.from_numpy(q2).to(DEV), torch.from_numpy(t).to(DEV), score_bits=8)
        bpbc.check_flags(0)


def test_error_flags_cover_every_stream():
    """A bad code scored on a side stream is reported by get_error_flags
    (which waits for this ctx's work on every stream it used)."""
    q, t = synth.gen_pairs(9002, 5000, 64, 64)
    t2 = t.copy()
    t2[4999, 63] = 200
    bpbc.get_error_flags(0)
    side = torch.cuda.Stream(DEV)
    dq, dt = torch.from_numpy(q).to(DEV), torch.from_numpy(t2).to(DEV)
    torch.cuda.synchronize()
    with torch.cuda.stream(side):
        bpbc.score_batch(dq, dt, score_bits=8, stream=side)
    assert bpbc.get_error_flags(0) & _lib.BPBC_FLAG_BAD_BASE


@pytest.mark.parametrize("pinned", [False, True])
@pytest.mark.parametrize("packed2", [False, True])
def test_host_path_chunks(pinned, packed2):
    """Host-buffer path with many chunks through the three slots, pageable
    or pinned output, u8 or 2-bit packed input; equal to the device path and
    to the oracle on a sample."""
    P, m, n = 300000, 64, 96
    q, t = synth.gen_pairs(9100, P, m, n, planted=True)
    out = (torch.empty(P, dtype=torch.int32, pin_memory=True).numpy() if pinned
           else np.empty(P, dtype=np.int32))
    for _ in range(2):  # the second call uses the rates the first measured
        if packed2:
            got = bpbc.score_batch_host_packed2(synth.pack2bit(q), synth.pack2bit(t), m, n,
                                                2, -1, -1, 8, out=out)
        else:
            got = bpbc.score_batch_host(q, t, 2, -1, -1, 8, out=out)
    dev = bpbc.score_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                           score_bits=8).cpu().numpy()
    np.testing.assert_array_equal(got, dev)
    idx = np.arange(0, P, 37)
    np.testing.assert_array_equal(got[idx], oracle.sw_batch(q[idx], t[idx], 2, -1, -1,
                                                            score_bits=8))


@pytest.mark.parametrize("P,m,n,packed2", [(600 * 32, 128, 1024, False), (650 * 32 - 5, 100, 4096, True),
                                           (32768, 128, 8192, False), (700 * 32, 200, 2048, False)])
def test_host_path_few_long_groups(P, m, n, packed2):
    """Host path of a wrap-around batch as one streamed launch (per-stream
    copy timelines moved in column blocks, the wrap kernel polling the wave
    count) matches the oracle; ragged P, padded rows, R = 8, 2-bit input."""
    q, t = synth.gen_pairs(9200 + n, P, m, n, planted=True)
    s = bpbc.default_score_bits(2, m, n)
    if packed2:
        got = bpbc.score_batch_host_packed2(synth.pack2bit(q), synth.pack2bit(t), m, n, 2, -1, -1, s)
    else:
        got = bpbc.score_batch_host(q, t, 2, -1, -1, s)
    plan = bpbc.last_plan(0)
    assert plan["wrap"] and plan["host_streamed"], plan
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=s))


def test_filter_on_side_stream():
    """filter_batch allocates its outputs on the stream it runs on."""
    q, t = synth.gen_pairs(9300, 4000, 64, 64, planted=True)
    side = torch.cuda.Stream(DEV)
    dq, dt = torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV)
    torch.cuda.synchronize()
    with torch.cuda.stream(side):
        mask, count, idx = bpbc.filter_batch(dq, dt, 60, score_bits=8, stream=side)
    side.synchronize()
    want = np.nonzero(oracle.sw_batch(q, t, 2, -1, -1) > 60)[0]
    c = int(count.item())
    assert c == want.size
    np.testing.assert_array_equal(idx.cpu().numpy()[:c], want)


def test_multi_device_driver_releases_ctxs_and_returns_flags():
    from paper_conf_ipps_nishimurabin17_b200 import parallel
    q, t = synth.gen_pairs(9400, 3000, 50, 70, planted=True)
    t2 = t.copy()
    t2[2999, 0] = 77  # in the last shard
    before = len(api._ctxs)
    got, flags = parallel.score_multi_device(q, t2, 2, -1, -1, 8, devices=[0, 0],
                                             return_flags=True)
    assert len(api._ctxs) == before  # worker ctxs were destroyed with their threads
    assert flags[1] & _lib.BPBC_FLAG_BAD_BASE and not flags[0]
    np.testing.assert_array_equal(got, oracle.sw_batch(q, t2 & 3, 2, -1, -1, score_bits=8))


@pytest.mark.parametrize("P,m,n,packed2", [(300000, 128, 128, False), (300000, 128, 128, True),
                                           (200001, 64, 100, False), (90000, 40, 1000, True),
                                           (150000, 200, 256, False)])
def test_host_streamed_launch(P, m, n, packed2):
    """bpbc_sw_score_batch_host as one streamed launch (waves copied on the
    copy stream, progress writes, the sweep polling them): equal to the
    device path; ragged P, n % 32 != 0 (chunks straddling a stream's
    consecutive -- strided -- groups), L = 16 and R = 8 tilings."""
    q, t = synth.gen_pairs(9500 + m + n, P, m, n, planted=True)
    s = bpbc.default_score_bits(2, m, n)
    if packed2:
        got = bpbc.score_batch_host_packed2(synth.pack2bit(q), synth.pack2bit(t), m, n, 2, -1, -1, s)
    else:
        got = bpbc.score_batch_host(q, t, 2, -1, -1, s)
    assert bpbc.last_plan(0)["host_streamed"]
    dev = bpbc.score_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                           score_bits=s).cpu().numpy()
    np.testing.assert_array_equal(got, dev)
    idx = np.arange(0, P, 53)
    np.testing.assert_array_equal(got[idx], oracle.sw_batch(q[idx], t[idx], 2, -1, -1, score_bits=s))


def test_host_chunked_knob_matches_streamed():
    """BPBC_CHUNKED_HOST=1 (a ctx made in a thread with it set) takes the
    chunked path; both give the oracle's scores."""
    import os
    import threading
    P, m, n = 120000, 96, 128
    q, t = synth.gen_pairs(9600, P, m, n, planted=True)
    box = {}

    def run():
        box["got"] = bpbc.score_batch_host(q, t, 2, -1, -1, 9)
        box["plan"] = bpbc.last_plan(0)
        bpbc.release_thread_ctx(0)

    os.environ["BPBC_CHUNKED_HOST"] = "1"
    try:
        th = threading.Thread(target=run)
        th.start()
        th.join()
    finally:
        os.environ.pop("BPBC_CHUNKED_HOST", None)
    assert not box["plan"]["host_streamed"]
    streamed = bpbc.score_batch_host(q, t, 2, -1, -1, 9)
    np.testing.assert_array_equal(box["got"], streamed)
    idx = np.arange(0, P, 41)
    np.testing.assert_array_equal(streamed[idx], oracle.sw_batch(q[idx], t[idx], 2, -1, -1,
                                                                 score_bits=9))


@pytest.mark.parametrize("s", [10, 12, 16])
def test_force_width_knob(s):
    """BPBC_FORCE_WIDTH=1 evaluates the circuit at score_bits (above s_exact
    the exact circuit is still exact): same scores, plan width = s."""
    import os
    import threading
    q, t = synth.gen_pairs(9700 + s, 5000, 64, 64, planted=True)
    box = {}

    def run():
        box["got"] = bpbc.score_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                                      score_bits=s).cpu().numpy()
        box["plan"] = bpbc.last_plan(0)
        bpbc.release_thread_ctx(0)

    os.environ["BPBC_FORCE_WIDTH"] = "1"
    try:
        th = threading.Thread(target=run)
        th.start()
        th.join()
    finally:
        os.environ.pop("BPBC_FORCE_WIDTH", None)
    assert box["plan"]["width"] == s
    np.testing.assert_array_equal(box["got"], oracle.sw_batch(q, t, 2, -1, -1, score_bits=s))


def test_host_path_under_launch_blocking(tmp_path):
    """With CUDA_LAUNCH_BLOCKING=1 a kernel cannot see a copy-stream write
    enqueued after its launch: the streamed host path's once-per-ctx probe
    (a 200 ms bounded wait) detects it and the call takes the chunked path --
    correct scores, no stall.  Runs in a subprocess, since the
    variable only takes effect at CUDA initialisation."""
    import os
    import subprocess
    import sys
    code = r'''
import sys, numpy as np
sys.path.insert(0, %r)
import oracle, synth
import paper_conf_ipps_nishimurabin17_b200 as bpbc
q, t = synth.gen_pairs(9900, 20000, 128, 128, planted=True)
got = bpbc.score_batch_host(q, t, 2, -1, -1, 9)
plan = bpbc.last_plan(0)
assert not plan["host_streamed"], plan
np.testing.assert_array_equal(got, oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))
assert bpbc.get_error_flags(0) == 0
print("OK")
''' % os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, CUDA_LAUNCH_BLOCKING="1")
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env,
                       timeout=600)
    assert r.returncode == 0 and "OK" in r.stdout, r.stdout[-2000:] + r.stderr[-2000:]
