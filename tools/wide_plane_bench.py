#!/usr/bin/env python3
"""GCUPS of one shape with given constants (no oracle): used for the
multi-warp wide-plane case (128 < m <= 256 at >= 13 bits), e.g.
    python tools/wide_plane_bench.py --pairs 524288 --m 200 --n 240 --consts 31,-1,-1 --s 13
"""
import argparse
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
import paper_conf_ipps_nishimurabin17_b200 as bpbc  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--pairs", type=int, default=1 << 19)
    ap.add_argument("--m", type=int, default=200)
    ap.add_argument("--n", type=int, default=240)
    ap.add_argument("--consts", default="31,-1,-1")
    ap.add_argument("--s", type=int, default=13)
    ap.add_argument("--steps", type=int, default=5)
    args = ap.parse_args()
    c = [int(x) for x in args.consts.split(",")]
    P, m, n = args.pairs, args.m, args.n
    q = np.empty((P, m), np.uint8)
    t = np.empty((P, n), np.uint8)
    synth.gen_pairs(1234, P, m, n, out_q=q, out_t=t)
    dq, dt = torch.from_numpy(q).cuda(), torch.from_numpy(t).cuda()
    out = torch.empty(P, dtype=torch.int32, device="cuda")
    ws = torch.empty(bpbc.workspace_bytes(P, m, n), dtype=torch.uint8, device="cuda")
    for _ in range(3):
        bpbc.score_batch(dq, dt, *c, score_bits=args.s, out=out, workspace=ws)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(args.steps):
        bpbc.score_batch(dq, dt, *c, score_bits=args.s, out=out, workspace=ws)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / args.steps
    print(f"P={P} m={m} n={n} consts={c} s={args.s}: {P * m * n / ms / 1e6:.1f} GCUPS, "
          f"{ms:.3f} ms, plan {bpbc.last_plan(0)}, checksum {int(out.sum().item())}")


if __name__ == "__main__":
    main()
