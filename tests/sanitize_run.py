#!/usr/bin/env python3
"""Small runs of every kernel family, for compute-sanitizer.

    compute-sanitizer --tool memcheck|racecheck|synccheck python tests/sanitize_run.py

Each case is small (sanitizers slow kernels ~100x) but spans several groups,
ragged pair counts and ragged lengths: the single-warp sweep (L = 16 and 32,
exact / saturating / runtime constants), the multi-warp sweep (shared-memory
boundary ring + phase barriers), the sequential striped sweep (global boundary
buffer), the threshold filter with compaction, the 2-bit packed input, the
wordwise comparator and the host path.  Every result is checked against the
oracle; exits non-zero on a mismatch.
"""
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))  # repo root
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_ipps_nishimurabin17_b200 as bpbc  # noqa: E402

DEV = "cuda:0"


def check(name, got, want):
    bad = int((np.asarray(got) != np.asarray(want)).sum())
    print(f"{name}: {'ok' if bad == 0 else f'{bad} MISMATCHES'}", flush=True)
    return bad


def main():
    bad = 0
    cases = [  # P, m, n, consts, s
        (97, 64, 80, (2, -1, -1), None),      # L = 16, exact
        (70, 128, 128, (2, -1, -1), None),    # L = 32, exact
        (40, 200, 230, (2, -1, -1), None),    # R = 8
        (50, 37, 61, (3, -2, -1), 12),        # runtime constants
        (50, 48, 80, (2, -1, -1), 5),         # saturating, fixed constants
        (33, 300, 320, (2, -1, -1), None),    # multi-warp W = 3 (4 groups per block)
        (20, 200, 240, (31, -1, -1), 13),     # multi-warp wide planes
        (9, 600, 640, (2, -1, -1), None),     # sequential stripes
        (40, 100, 130, (3, -2, -2), None),    # exact circuit, runtime constants
        (33, 300, 320, (1, -1, -1), None),    # ... multi-warp W = 3
        (9, 600, 640, (1, -3, -5), None),     # ... sequential stripes
    ]
    for P, m, n, (c1, mm, g), s in cases:
        q, t = synth.gen_pairs(4000 + m + n, P, m, n, planted=True)
        s = s or bpbc.default_score_bits(c1, m, n)
        got = bpbc.score_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV), c1, mm, g,
                               score_bits=s).cpu().numpy()
        bad += check(f"score P={P} m={m} n={n} c={c1},{mm},{g} s={s} plan={bpbc.last_plan(0)}",
                     got, oracle.sw_batch(q, t, c1, mm, g, score_bits=s))
    # threshold filter with compaction
    q, t = synth.gen_pairs(77, 150, 64, 96, planted=True)
    mask, count, idx = bpbc.filter_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV), 40)
    want = np.nonzero(oracle.sw_batch(q, t, 2, -1, -1) > 40)[0]
    c = int(count.item())
    # only the first count entries are written (bpbc_sw.h): copy just those
    bad += check("filter indices", idx[:c].cpu().numpy(), want)
    # packed2 input, wordwise comparator, host path
    q, t = synth.gen_pairs(78, 90, 72, 100, planted=True)
    want = oracle.sw_batch(q, t, 2, -1, -1, score_bits=9)
    got = bpbc.score_batch_packed2(torch.from_numpy(synth.pack2bit(q)).to(DEV),
                                   torch.from_numpy(synth.pack2bit(t)).to(DEV), 72, 100,
                                   score_bits=9).cpu().numpy()
    bad += check("packed2", got, want)
    got = bpbc.score_batch_wordwise(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV)).cpu()
    bad += check("wordwise", got.numpy(), oracle.sw_batch(q, t, 2, -1, -1))
    bad += check("host path", bpbc.score_batch_host(q, t, 2, -1, -1, 9), want)
    # wrap-around schedule (snapshot hand-off through global memory with
    # acquire/release flags), forced on a 600-group batch in a thread whose
    # ctx reads BPBC_WRAP=1 / one block per SM at init
    q, t = synth.gen_pairs(79, 600 * 32, 128, 256, planted=True)
    res = {}

    def wrap_case():
        res["got"] = bpbc.score_batch(torch.from_numpy(q).to(DEV), torch.from_numpy(t).to(DEV),
                                      score_bits=9).cpu().numpy()
        res["plan"] = bpbc.last_plan(0)
        bpbc.release_thread_ctx(0)

    os.environ.update({"BPBC_WRAP": "1", "BPBC_MAX_BLOCKS_PER_SM": "1"})
    th = threading.Thread(target=wrap_case)
    th.start()
    th.join()
    for k in ("BPBC_WRAP", "BPBC_MAX_BLOCKS_PER_SM"):
        os.environ.pop(k, None)
    bad += check(f"wrap-around plan={res.get('plan')}", res.get("got"),
                 oracle.sw_batch(q, t, 2, -1, -1, score_bits=9))
    # two streams through one ctx with the ctx-owned workspace (workspace =
    # NULL): the second call waits for the first one's use of it
    qa, ta = synth.gen_pairs(80, 300, 64, 64, planted=True)
    qb, tb = synth.gen_pairs(81, 500, 64, 96, planted=True)
    s1, s2 = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    da = [torch.from_numpy(x).to(DEV) for x in (qa, ta)]
    db = [torch.from_numpy(x).to(DEV) for x in (qb, tb)]
    torch.cuda.synchronize()
    with torch.cuda.stream(s1):
        oa = bpbc.score_batch(*da, score_bits=8, stream=s1)
    with torch.cuda.stream(s2):
        ob = bpbc.score_batch(*db, score_bits=8, stream=s2)
    torch.cuda.synchronize()
    bad += check("two streams, ctx workspace (a)", oa.cpu().numpy(),
                 oracle.sw_batch(qa, ta, 2, -1, -1, score_bits=8))
    bad += check("two streams, ctx workspace (b)", ob.cpu().numpy(),
                 oracle.sw_batch(qb, tb, 2, -1, -1, score_bits=8))
    # the standalone transpose kernel (W2B) against its definition
    codes = np.random.default_rng(5).integers(0, 4, size=(70, 300), dtype=np.uint8)
    planes = bpbc.pack(torch.from_numpy(codes).to(DEV)).cpu().numpy().view(np.uint32)
    bad += check("pack", planes, oracle.pack_planes(codes))
    torch.cuda.synchronize()
    print("sanitize_run:", "PASS" if bad == 0 else "FAIL", flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
