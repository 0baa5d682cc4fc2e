#!/usr/bin/env python3
"""The paper's own workload on one B200, in the layout of its Table IV
(H2G / W2B / SWA / B2W / G2H milliseconds per n): 32768 pairs,
m = 128, n = 1024 ... 65536, +2/-1/-1, 9-bit slices.

usage: python tools/paper_table.py [--n 1024,2048,...] [--steps 5] [--out profiles/r2_paper_table]

Per n (inputs generated into pinned host memory, seeded):
  H2G   CUDA-event time of the pinned host->device copy of the u8 query and
        target rows;
  W2B   the standalone transpose kernel bpbc_sw_pack of query and target
         -- the hot path runs it FUSED into the sweep (its cost is
        inside SWA); shown for the paper's column;
  SWA   the sweep kernel (with the fused W2B), from the library's
        own CUDA events on its stream (bpbc_sw_profile);
  B2W   the max-reduction + untranspose kernel;
  G2H   the device->host copy of the 32768 int32 scores;
  total = H2G + SWA + B2W + G2H; kernel GCUPS = cells / (SWA + B2W);
  e2e   bpbc_sw_score_batch_host wall time (H2D, kernels and D2H overlapped
        by the 3-slot host path);
plus the sweep's fraction of the measured LOP3 peak and the paper's TITAN X
numbers for the same n (context only).  Timing rules as
bench.py (3 warm-ups, CUDA events, 256 MiB L2 flush between steps, clocks).
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

import bench  # noqa: E402
import synth  # noqa: E402
import paper_conf_ipps_nishimurabin17_b200 as bpbc  # noqa: E402

P, M, S = 32768, 128, 9
# Table IV GPU bitwise-32 rows, ms: H2G, W2B, SWA, B2W, G2H, total
PAPER = {1024: (5.51, 0.14, 6.91, 0.01, 0.08, 12.66), 65536: (299.47, 3.35, 392.52, 0.01, 0.08, 695.42)}


def ev_time(fn, steps, flush):
    return bench.time_device_steps(fn, steps, 3, flush) / steps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", default="1024,2048,4096,8192,16384,32768,65536")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2_paper_table"))
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    peak, peak_src = bench.measured_lop3_peak()
    rows = []
    sampler = bench.ClockSampler(0).start()
    for n in [int(x) for x in a.n.split(",")]:
        hq = torch.empty((P, M), dtype=torch.uint8, pin_memory=True)
        ht = torch.empty((P, n), dtype=torch.uint8, pin_memory=True)
        synth.gen_pairs(synth.seed_for_config(6) + n, P, M, n, out_q=hq.numpy(), out_t=ht.numpy())
        dq = torch.empty((P, M), dtype=torch.uint8, device=dev)
        dt = torch.empty((P, n), dtype=torch.uint8, device=dev)
        out = torch.empty(P, dtype=torch.int32, device=dev)
        hout = torch.empty(P, dtype=torch.int32, pin_memory=True)
        h2g = ev_time(lambda: (dq.copy_(hq, non_blocking=True), dt.copy_(ht, non_blocking=True)),
                      a.steps, flush)
        ws = torch.empty(bpbc.workspace_bytes_for(P, M, n, 2, -1, -1, score_bits=S),
                         dtype=torch.uint8, device=dev)
        G = (P + 31) // 32
        pq = torch.empty((G, M, 2), dtype=torch.int32, device=dev)
        pt = torch.empty((G, n, 2), dtype=torch.int32, device=dev)
        w2b = ev_time(lambda: (bpbc.pack(dq, out=pq), bpbc.pack(dt, out=pt)), a.steps, flush)
        del pq, pt
        step = lambda: bpbc.score_batch(dq, dt, 2, -1, -1, score_bits=S, out=out, workspace=ws)
        for _ in range(3):
            step()
        torch.cuda.synchronize()
        bpbc.profile(True, 0)
        dev_ms = ev_time(step, a.steps, flush)
        ph = bpbc.profile_read(0)
        bpbc.profile(False, 0)
        plan = bpbc.last_plan(0)
        c = max(1, ph["calls"])
        swa, b2w = ph["swa_ms"] / c, ph["b2w_ms"] / c
        g2h = ev_time(lambda: hout.copy_(out, non_blocking=True), a.steps, flush)
        # end to end through the host-buffer C call
        qn, tn, on = hq.numpy(), ht.numpy(), hout.numpy()
        for _ in range(2):
            bpbc.score_batch_host(qn, tn, 2, -1, -1, S, out=on)
        t0 = time.perf_counter()
        for _ in range(a.steps):
            bpbc.score_batch_host(qn, tn, 2, -1, -1, S, out=on)
        e2e_ms = (time.perf_counter() - t0) / a.steps * 1e3
        assert np.array_equal(on, out.cpu().numpy())
        cells = P * M * n
        frac = plan["ops_per_word_cell"] * (G * M * n) / (swa / 1e3) / 1e12 / peak
        total = h2g + swa + b2w + g2h
        row = {"n": n, "H2G_ms": h2g, "W2B_ms_standalone": w2b, "SWA_ms": swa, "B2W_ms": b2w,
               "G2H_ms": g2h, "total_ms": total, "device_step_ms": dev_ms, "e2e_ms": e2e_ms,
               "kernel_gcups": cells / ((swa + b2w) / 1e3) / 1e9,
               "device_gcups": cells / (dev_ms / 1e3) / 1e9,
               "total_gcups": cells / (total / 1e3) / 1e9, "e2e_gcups": cells / (e2e_ms / 1e3) / 1e9,
               "sweep_frac_lop3_peak": frac, "plan": plan}
        if n in PAPER:
            row["paper_titanx_ms"] = dict(zip(["H2G", "W2B", "SWA", "B2W", "G2H", "total"], PAPER[n]))
        rows.append(row)
        print(json.dumps(row), flush=True)
        del hq, ht, dq, dt, ws
        torch.cuda.empty_cache()
    clocks = sampler.stop()
    md = ["| n | H2G ms | W2B ms (standalone; fused in SWA) | SWA ms | B2W ms | G2H ms | total ms | "
          "kernel GCUPS | e2e ms (overlapped host path) | e2e GCUPS | sweep frac of LOP3 peak | schedule |",
          "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in rows:
        md.append(f"| {r['n']} | {r['H2G_ms']:.2f} | {r['W2B_ms_standalone']:.3f} | {r['SWA_ms']:.2f} | "
                  f"{r['B2W_ms']:.3f} | {r['G2H_ms']:.3f} | {r['total_ms']:.2f} | {r['kernel_gcups']:.0f} | "
                  f"{r['e2e_ms']:.2f} | {r['e2e_gcups']:.0f} | {r['sweep_frac_lop3_peak']:.3f} | "
                  f"{'wrap-around' if r['plan']['wrap'] else 'group-granular'}, {r['plan']['streams']} streams, "
                  f"{r['plan']['blocks_per_sm']} block/SM |")
    md.append("")
    md.append(f"Clocks during the run: {clocks}. Peak: {peak:.2f} T LOP3 lane-ops/s ({peak_src}).")
    md.append("Paper (TITAN X, P:L393-399, context only): n=1024 H2G 5.51 / W2B 0.14 / SWA 6.91 / "
              "B2W 0.01 / G2H 0.08 = 12.66 ms; n=65536 299.47 / 3.35 / 392.52 / 0.01 / 0.08 = 695.42 ms.")
    open(a.out + ".md", "w").write("\n".join(md) + "\n")
    json.dump({"rows": rows, "clocks": clocks, "peak": peak, "peak_source": peak_src},
              open(a.out + ".json", "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
