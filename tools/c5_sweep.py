#!/usr/bin/env python3
"""BASELINE config 5 on one B200: GCUPS vs score width s = 6..12 and length
m = n = 32..512 (2^22 pairs per point, +2/-1/-1), with the sweep kernel's
fraction of the LOP3 peak and the share of outputs capped at 2^s - 1 (R3).

usage: python tools/c5_sweep.py [--pairs 4194304] [--steps 5] [--warmup 3]
                                [--m 32,64,...] [--s 6,7,...] [--out FILE]

Same timing rules as bench.py (inputs resident in HBM, 256 MiB L2 flush
between steps, CUDA events, clocks sampled during the timed region).  One
input batch per m is shared by every s (one seed per m), so
out(s) = min(out(s'), 2^s - 1) must hold across the widths of a point; the
script checks that law on the GPU results (bit-exact parity of these points
against the oracle is in tests/test_gpu_parity.py).  Prints a markdown table
and writes the points as JSON.
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402  (CONSTS, peak, clock sampler)
import synth  # noqa: E402
import paper_conf_ipps_nishimurabin17_b200 as bpbc  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--pairs", type=int, default=1 << 22)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--m", default="32,64,128,256,512")
    ap.add_argument("--s", default="6,7,8,9,10,11,12")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "c5_sweep.json"))
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    P = args.pairs
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    points = []
    for m in [int(x) for x in args.m.split(",")]:
        n = m
        seed = synth.seed_for_config(5) + int(np.log2(m))
        hq = np.empty((P, m), dtype=np.uint8)
        ht = np.empty((P, n), dtype=np.uint8)
        synth.gen_pairs(seed, P, m, n, out_q=hq, out_t=ht)
        dq = torch.from_numpy(hq).to(dev)
        dt = torch.from_numpy(ht).to(dev)
        del hq, ht
        out = torch.empty(P, dtype=torch.int32, device=dev)
        ws = torch.empty(bpbc.workspace_bytes(P, m, n), dtype=torch.uint8, device=dev)
        widest = None
        for s in sorted([int(x) for x in args.s.split(",")], reverse=True):
            def step():
                bpbc.score_batch(dq, dt, *bench.CONSTS, score_bits=s, out=out, workspace=ws)

            for _ in range(args.warmup):
                step()
            torch.cuda.synchronize()
            plan = bpbc.last_plan(0)
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                  for _ in range(args.steps)]
            sampler = bench.ClockSampler(0).start()
            time.sleep(0.3)
            bpbc.profile(True, 0)
            for a, b in ev:
                flush.zero_()
                a.record()
                step()
                b.record()
            torch.cuda.synchronize()
            clocks = sampler.stop()
            ph = bpbc.profile_read(0)
            bpbc.profile(False, 0)
            t_ms = sum(a.elapsed_time(b) for a, b in ev)
            gcups = P * m * n * args.steps / (t_ms / 1e3) / 1e9
            sweep_ms = ph["swa_ms"] / max(1, ph["calls"])
            word_cells = (P + 31) // 32 * m * n
            peak = bench.measured_lop3_peak()[0]
            frac = plan["ops_per_word_cell"] * word_cells / (sweep_ms / 1e3) / 1e12 / peak
            got = out.cpu().numpy()
            cap = (1 << s) - 1
            if widest is None:
                widest = (s, got.copy())
                law = True
            else:  # cross-width law (R3) against the widest width of this m
                law = bool(np.array_equal(got, np.minimum(widest[1], cap)))
            pt = {"m": m, "n": n, "s": s, "pairs": P, "gcups": round(gcups, 1),
                  "ms_per_step": round(t_ms / args.steps, 3), "sweep_ms": round(sweep_ms, 3),
                  "frac_lop3_peak": round(frac, 4), "plan": plan,
                  "saturated_frac": round(float((got == cap).mean()), 6),
                  "mean_score": round(float(got.mean()), 2), "max_score": int(got.max()),
                  "cross_width_law": law, "clocks": clocks}
            points.append(pt)
            print(json.dumps(pt), flush=True)
        del dq, dt, out, ws
        torch.cuda.empty_cache()
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump({"what": "C5 sweep on 1 B200 (tools/c5_sweep.py)", "points": points},
              open(args.out, "w"), indent=1)
    ms = sorted({p["m"] for p in points})
    ss = sorted({p["s"] for p in points})
    get = {(p["m"], p["s"]): p for p in points}
    print("\n| m = n | " + " | ".join(f"s={s}" for s in ss) + " |")
    print("|---|" + "---|" * len(ss))
    for m in ms:
        cells = []
        for s in ss:
            p = get.get((m, s))
            cells.append("—" if p is None else
                         f"{p['gcups']:.0f} ({p['frac_lop3_peak']:.2f}, sat {p['saturated_frac']:.2f})")
        print(f"| {m} | " + " | ".join(cells) + " |")
    bad = [p for p in points if not p["cross_width_law"]]
    print(f"\ncross-width law violations: {len(bad)}")
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
