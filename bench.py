#!/usr/bin/env python3
"""bench.py -- BPBC Smith-Waterman on B200: GCUPS with bit-exact max local scores.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2] [--impl ours|reference]

One "step" = the whole hot path (W2B pack of query and target -> bit-sliced
wavefront sweep -> max reduction + B2W untranspose) over one
batch of synthetic pairs already resident in HBM.  Default workload (N=1) is
BASELINE.json configs[1] = C2: 2^20 DNA pairs, m = n = 128, +2/-1/-1, 9-bit
slices.  For N > 1 (torchrun, one process per GPU) every rank scores its own
C2-sized shard (weak scaling, no collective on the data path); the int32
scores are all-gathered once after the timed region.

Prints ONE JSON line on rank 0 (contract in the task statement / DESIGN.md
"Measurement"): metric, value (GCUPS, all ranks), e2e (same metric through
the host-buffer C call bpbc_sw_score_batch_host with pinned host inputs,
H2D + D2H inside the timed region), roofline (the sweep kernel against the
integer-logic pipe peak), cpu_baseline (the oracle on a bounded sample on
this host's cores), clocks (nvidia-smi sampled during the timed region),
gpu_launches, parity (the GPU scores of the cpu_baseline sample checked
against the oracle's; N=1 only, like cpu_baseline).

--impl reference times the CPU oracle (oracle/) on the same config -- the
reference arm of this tier (no reference implementation exists).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "GCUPS (bit-exact max local score)"
CONFIGS = {  # BASELINE.json configs; "scaling" says how N GPUs split it
    1: dict(P=1024, m=64, n=64, s=8, scaling="weak"),
    2: dict(P=1 << 20, m=128, n=128, s=9, scaling="weak"),
    3: dict(P=1 << 22, m=256, n=256, s=10, scaling="strong"),  # 2^22 pairs sharded over N
    4: dict(P=1 << 20, m=64, n=1024, s=8, scaling="weak"),
    5: dict(P=1 << 22, m=512, n=512, s=11, scaling="weak"),  # one point of the C5 sweep
    6: dict(P=32768, m=128, n=65536, s=9, scaling="weak"),  # the paper's own shape
}
CONSTS = (2, -1, -1)  # match, mismatch, gap (Table II, reading R14)
SM_COUNT = 148
ALU_LANES_PER_SM_CLK = 64  # 4 SMSP x 16 lanes/clk (LOP3 rt = 2 cyc per warp instr)


def workload_name(cid, c):
    name = "paper shape (P:L382)" if cid == 6 else f"C{cid}"
    return (f"{name}: {c['P']} DNA pairs, m={c['m']}, n={c['n']}, "
            f"match/mismatch/gap = +2/-1/-1, {c['s']}-bit score slices, max score only")


def survey_ops_per_word_cell(s):
    """LOP3 form of the circuit, 11s + 2 per 32-cell word."""
    return 11 * s + 2


def peak_alu_tops(sm_mhz):
    return SM_COUNT * ALU_LANES_PER_SM_CLK * sm_mhz * 1e6 / 1e12


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.thread.join(timeout=2)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_baseline(cfg, target_seconds=12.0):
    """The oracle as it stands, on a bounded sample of the workload (its first
    pairs), all host cores.  Returns the cpu_baseline object and the oracle's
    scores of the sample, which the caller compares with the GPU's (parity)."""
    import oracle
    import synth
    threads = os.cpu_count() or 1
    m, n = cfg["m"], cfg["n"]
    seed = synth.seed_for_config(cfg["id"])
    # calibrate the rate on a warm library with enough pairs per thread that
    # thread start-up does not dominate, then size the sample to ~target_seconds
    cal = int(min(cfg["P"], max(64 * threads, 4096)))
    q, t = synth.gen_pairs(seed, cal, m, n)
    oracle.sw_batch(q[:threads], t[:threads], *CONSTS, score_bits=cfg["s"], threads=threads)
    t0 = time.perf_counter()
    oracle.sw_batch(q, t, *CONSTS, score_bits=cfg["s"], threads=threads)
    rate = cal / max(time.perf_counter() - t0, 1e-6)
    sample = int(min(cfg["P"], max(cal, rate * target_seconds)))
    q, t = synth.gen_pairs(seed, sample, m, n)
    t0 = time.perf_counter()
    want = oracle.sw_batch(q, t, *CONSTS, score_bits=cfg["s"], threads=threads)
    dt = time.perf_counter() - t0
    return {"value": round(sample * m * n / dt / 1e9, 4), "unit": "GCUPS", "cores": threads,
            "kind": "oracle",
            "sample": f"first {sample} of the {cfg['P']} pairs of C{cfg['id']} "
                      f"(m={m}, n={n}), {dt:.1f} s, scalar int32 DP, {threads} threads"}, want


def run_reference(args, cfg):
    """--impl reference: the CPU oracle timed on this host (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    import synth
    threads = os.cpu_count() or 1
    m, n = cfg["m"], cfg["n"]
    seed = synth.seed_for_config(cfg["id"])
    # size one step so the whole run stays within ~1-2 minutes
    cal = int(min(cfg["P"], max(64 * threads, 4096)))
    q, t = synth.gen_pairs(seed, cal, m, n)
    oracle.sw_batch(q[:threads], t[:threads], *CONSTS, score_bits=cfg["s"], threads=threads)
    t0 = time.perf_counter()
    oracle.sw_batch(q, t, *CONSTS, score_bits=cfg["s"], threads=threads)
    rate = cal / max(time.perf_counter() - t0, 1e-6)
    per_step = int(min(cfg["P"], max(threads, rate * 60.0 / max(1, args.steps + args.warmup))))
    q, t = synth.gen_pairs(seed, per_step, m, n)
    for _ in range(args.warmup):
        oracle.sw_batch(q, t, *CONSTS, score_bits=cfg["s"], threads=threads)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.sw_batch(q, t, *CONSTS, score_bits=cfg["s"], threads=threads)
    dt = time.perf_counter() - t0
    v = per_step * m * n * args.steps / dt / 1e9
    line = {"metric": METRIC, "value": round(v, 4), "unit": "GCUPS", "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(dt / args.steps * 1e3, 3), "higher_is_better": True,
            "scaling": cfg["scaling"], "vs_baseline": None, "dtype": "int32",
            "data": "synthetic",
            "config": {"workload": workload_name(cfg["id"], cfg),
                       "sample_pairs_per_step": per_step},
            "cpu_baseline": {"value": round(v, 4), "unit": "GCUPS", "cores": threads,
                             "kind": "oracle",
                             "sample": f"{per_step} pairs of C{cfg['id']} per step"},
            "e2e": {"value": round(v, 4), "unit": "GCUPS", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=2, choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--score-bits", type=int, default=None)
    ap.add_argument("--m", type=int, default=None, help="override the query length")
    ap.add_argument("--n", type=int, default=None, help="override the target length")
    ap.add_argument("--pairs", type=int, default=None, help="override the pair count")
    ap.add_argument("--no-filter", action="store_true")
    ap.add_argument("--filter-threshold", type=int, default=None,
                    help="tau of the threshold-filter line (default 0.9 * min(m, n))")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    cfg = dict(CONFIGS[args.config])
    cfg["id"] = args.config
    if args.score_bits:
        cfg["s"] = args.score_bits
    for key, val in (("m", args.m), ("n", args.n), ("P", args.pairs)):
        if val:
            cfg[key] = val
    if args.impl == "reference":
        run_reference(args, cfg)
        return

    import torch
    import torch.distributed as dist

    import synth
    import paper_conf_ipps_nishimurabin17_b200 as bpbc

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ngpu = torch.cuda.device_count()
    # More ranks than GPUs (only for exercising the N > 1 code path on a
    # 1-GPU box): ranks share devices and the collectives go through gloo on
    # the host; the timing is then not a scaling measurement.
    shared = world > ngpu
    if shared:
        local = local % max(1, ngpu)
    if world > 1:
        torch.cuda.set_device(local)
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    cdev = torch.device("cpu") if shared else dev  # where collective tensors live
    torch.cuda.set_device(dev)
    m, n, s = cfg["m"], cfg["n"], cfg["s"]
    seed = synth.seed_for_config(args.config)
    from paper_conf_ipps_nishimurabin17_b200 import parallel
    if cfg["scaling"] == "strong":  # the config's pairs split over the ranks
        P_total = cfg["P"]
        p0, p1 = parallel.shard_range(P_total, world, rank)
    else:  # every rank scores a config-sized batch of its own
        P_total = world * cfg["P"]
        p0, p1 = rank * cfg["P"], (rank + 1) * cfg["P"]
    P = p1 - p0

    # inputs: this rank's shard, generated on the host into pinned buffers
    hq = torch.empty((P, m), dtype=torch.uint8, pin_memory=True)
    ht = torch.empty((P, n), dtype=torch.uint8, pin_memory=True)
    synth.gen_pairs(seed, P, m, n, p_offset=p0, out_q=hq.numpy(), out_t=ht.numpy())
    dq = hq.to(dev, non_blocking=True)
    dt = ht.to(dev, non_blocking=True)
    out = torch.empty(P, dtype=torch.int32, device=dev)
    ws = torch.empty(bpbc.workspace_bytes(P, m, n), dtype=torch.uint8, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    torch.cuda.synchronize()

    def step():
        # the whole hot path on this rank's shard; no collective on the data
        # path (pairs are independent)
        bpbc.score_batch(dq, dt, *CONSTS, score_bits=s, out=out, workspace=ws)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    plan = bpbc.last_plan(local)

    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    sampler = ClockSampler(local).start()
    time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    bpbc.profile(True, local)
    for k in range(args.steps):
        flush.zero_()  # L2 flush between timed steps (outside the events)
        starts[k].record()
        step()
        ends[k].record()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    phases = bpbc.profile_read(local)
    bpbc.profile(False, local)
    t_ms = sum(a.elapsed_time(b) for a, b in zip(starts, ends))
    if world > 1:
        tt = torch.tensor([t_ms], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_ms = tt.item()
    cells = P_total * m * n * args.steps
    gcups = cells / (t_ms / 1e3) / 1e9

    # ---------------- threshold filter (NEXT-2) on the same resident batch
    filt = None
    if not args.no_filter:
        tau = args.filter_threshold if args.filter_threshold is not None else int(0.9 * min(m, n))
        fmask = torch.empty((P + 31) // 32, dtype=torch.int32, device=dev)
        fidx = torch.empty(P, dtype=torch.int64, device=dev)
        fcnt = torch.zeros(1, dtype=torch.int64, device=dev)

        def fstep():
            bpbc.filter_batch(dq, dt, tau, *CONSTS, score_bits=s, workspace=ws)

        for _ in range(args.warmup):
            fstep()
        fk = max(3, min(args.steps, 10))
        fs = [torch.cuda.Event(enable_timing=True) for _ in range(fk)]
        fe = [torch.cuda.Event(enable_timing=True) for _ in range(fk)]
        torch.cuda.synchronize()
        for k in range(fk):
            flush.zero_()
            fs[k].record()
            fstep()
            fe[k].record()
        torch.cuda.synchronize()
        f_ms = sum(x.elapsed_time(y) for x, y in zip(fs, fe))
        _, cnt, _ = bpbc.filter_batch(dq, dt, tau, *CONSTS, score_bits=s, workspace=ws)
        filt = {"value": round(P * m * n * fk / (f_ms / 1e3) / 1e9, 2), "unit": "GCUPS",
                "threshold": tau, "flagged_pairs_rank0": int(cnt.item()),
                "ms_per_step": round(f_ms / fk, 4),
                "what": "bpbc_sw_filter_batch: pairs with max score > threshold, mask + "
                        "ascending indices (P:L231)"}
        del fmask, fidx, fcnt

    # ---------------- wordwise comparator (NEXT-4) on the same resident batch
    wordwise = None
    if not args.no_filter and min(m, n) <= 256:
        wout = torch.empty(P, dtype=torch.int32, device=dev)

        def wstep():
            bpbc.score_batch_wordwise(dq, dt, *CONSTS, out=wout)

        for _ in range(args.warmup):
            wstep()
        wk = max(3, min(args.steps, 10))
        ws0 = [torch.cuda.Event(enable_timing=True) for _ in range(wk)]
        ws1 = [torch.cuda.Event(enable_timing=True) for _ in range(wk)]
        torch.cuda.synchronize()
        for k in range(wk):
            flush.zero_()
            ws0[k].record()
            wstep()
            ws1[k].record()
        torch.cuda.synchronize()
        w_ms = sum(x.elapsed_time(y) for x, y in zip(ws0, ws1))
        wv = P * m * n * wk / (w_ms / 1e3) / 1e9
        cap = (1 << s) - 1
        agree = bool(torch.equal(torch.clamp(wout, max=cap), out))
        wordwise = {"value": round(wv, 2), "unit": "GCUPS", "ms_per_step": round(w_ms / wk, 4),
                    "bitwise_over_wordwise": round(gcups / world / wv, 3) if wv else None,
                    "agrees_with_bitwise": agree,
                    "what": "bpbc_sw_score_batch_wordwise: ordinary-integer DP, 16-bit SIMD, "
                            "2 pairs per warp register (the paper's GPU wordwise row, P:L407)"}
        del wout

    # ---------------- end to end through the host-buffer C call
    e2e = e2e_packed2 = None
    if not args.no_e2e:
        hout = torch.empty(P, dtype=torch.int32, pin_memory=True)
        qn, tn, on = hq.numpy(), ht.numpy(), hout.numpy()
        for _ in range(2):
            bpbc.score_batch_host(qn, tn, *CONSTS, score_bits=s, device=local, out=on)
        if world > 1:
            dist.barrier()
        ksteps = max(3, min(args.steps, 10))
        t0 = time.perf_counter()
        for _ in range(ksteps):
            bpbc.score_batch_host(qn, tn, *CONSTS, score_bits=s, device=local, out=on)
        el = time.perf_counter() - t0
        if world > 1:
            te = torch.tensor([el], dtype=torch.float64, device=cdev)
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            el = te.item()
        e2e = {"value": round(P_total * m * n * ksteps / el / 1e9, 2), "unit": "GCUPS",
               "h2d_bytes_per_step": P_total * (m + n), "d2h_bytes_per_step": P_total * 4,
               "steps": ksteps, "timing": "host wall clock around the blocking C call "
                                          "bpbc_sw_score_batch_host (pinned host buffers, "
                                          "1 byte per base)"}
        # same through bpbc_sw_score_batch_host_packed2 (2-bit packed host
        # rows, 4x fewer H2D bytes; packing is input preparation, untimed)
        hq2 = torch.from_numpy(synth.pack2bit(hq.numpy())).pin_memory()
        ht2 = torch.from_numpy(synth.pack2bit(ht.numpy())).pin_memory()
        q2n, t2n = hq2.numpy(), ht2.numpy()
        for _ in range(2):
            bpbc.score_batch_host_packed2(q2n, t2n, m, n, *CONSTS, score_bits=s, device=local,
                                          out=on)
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(ksteps):
            bpbc.score_batch_host_packed2(q2n, t2n, m, n, *CONSTS, score_bits=s, device=local,
                                          out=on)
        el2 = time.perf_counter() - t0
        if world > 1:
            te = torch.tensor([el2], dtype=torch.float64, device=cdev)
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            el2 = te.item()
        e2e_packed2 = {"value": round(P_total * m * n * ksteps / el2 / 1e9, 2), "unit": "GCUPS",
                       "h2d_bytes_per_step": P_total * ((m + 3) // 4 + (n + 3) // 4),
                       "d2h_bytes_per_step": P_total * 4, "steps": ksteps,
                       "timing": "host wall clock around bpbc_sw_score_batch_host_packed2 "
                                 "(pinned, 2-bit packed bases)"}

    # ---------------- result gather (outside the timed region)
    if world > 1:  # rank r holds the pairs of shard_range(P_total, world, r)
        full = parallel.gather_scores(out.to(cdev), P_total)
        got_all = full.cpu().numpy()
    else:
        got_all = out.cpu().numpy()
    if rank != 0:
        dist.destroy_process_group()
        return

    # ---------------- roofline of the sweep kernel (integer-logic pipe)
    calls = max(1, phases["calls"])
    sweep_ms = phases["swa_ms"] / calls
    word_cells = (P + 31) // 32 * m * n
    # algorithmic LOP3 per word-cell = hand count of the circuit the plan
    # evaluates; SURVEY's 11s+2 is printed beside it
    alg_ops = plan["ops_per_word_cell"] * word_cells
    achieved = alg_ops / (sweep_ms / 1e3) / 1e12
    sm_max = clocks.get("sm_max_mhz") or 1965.0
    peak = peak_alu_tops(sm_max)
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get(f"C{args.config}", {}).get("sweep_dram_bytes")
        except Exception:
            traffic = None
    roofline = {"bound": "alu", "achieved": round(achieved, 3), "peak": round(peak, 3),
                "unit": "Tops/s (LOP3 lane-ops)", "frac": round(achieved / peak, 4),
                "traffic": traffic, "kernel": "sw_sweep_kernel",
                "kernel_ms_per_launch": round(sweep_ms, 4),
                "alg_ops_per_word_cell": plan["ops_per_word_cell"],
                "alg_ops_per_word_cell_survey": survey_ops_per_word_cell(s),
                "word_cells_per_launch": word_cells,
                "peak_basis": f"{SM_COUNT} SMs x {ALU_LANES_PER_SM_CLK} LOP3 lanes/clk x "
                              f"{sm_max:.0f} MHz (B300_MICROARCH alu rt=2/SMSP)",
                "phase_ms_per_step": {k: round(v / calls, 4) for k, v in phases.items()
                                      if k.endswith("_ms")}}
    # W2B (pack_kernel) against the measured HBM copy bandwidth, when the plan
    # runs it (multi-warp, striped and short-target plans); the fused sweep
    # transposes the raw codes itself and has no W2B launch
    w2b = None
    w2b_ms = phases.get("w2b_ms", 0.0) / calls
    if not plan.get("fused") and w2b_ms > 0:
        hbm = 6552.0
        try:
            hbm = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
            hbm_src = "MEASURED_PEAKS.json hbm_gbs"
        except Exception:
            hbm_src = "fallback 6552 GB/s (MEASURED_PEAKS.json unreadable)"
        mq, nt = min(m, n), max(m, n)
        groups = (P + 31) // 32
        nbytes = P * (m + n) + 8 * groups * (mq + nt)  # u8 codes read + uint2 planes written
        gbs = nbytes / (w2b_ms / 1e3) / 1e9
        w2b = {"bound": "hbm", "kernel": "pack_kernel", "achieved": round(gbs, 1),
               "peak": hbm, "unit": "GB/s", "frac": round(gbs / hbm, 4),
               "bytes_per_launch": nbytes, "ms_per_launch": round(w2b_ms, 4),
               "peak_source": hbm_src}

    cpu = None
    parity = None
    if not args.no_cpu_baseline and world == 1:
        # the cpu_baseline leg's oracle scores of the first pairs double as the
        # bench's bit-exact parity check of the GPU results for those pairs
        cpu, want = cpu_baseline(cfg)
        parity = {"pairs_checked": int(want.size),
                  "mismatches": int((got_all[:want.size] != want).sum()),
                  "what": "GPU scores of the cpu_baseline sample vs the oracle's"}
    # score distribution of the batch (C5: the share capped at 2^s - 1, R3)
    scores = {"mean": round(float(got_all.mean()), 3), "max": int(got_all.max()),
              "saturated_frac": round(float((got_all == (1 << s) - 1).mean()), 6)}

    line = {"metric": METRIC, "value": round(gcups, 2), "unit": "GCUPS", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(t_ms / args.steps, 4), "higher_is_better": True,
            "scaling": cfg["scaling"], "vs_baseline": None,
            "dtype": "u32 bit-sliced (s-bit scores)",
            "data": "synthetic (seeded i.i.d. uniform DNA, SplitMix64)",
            "config": {"workload": workload_name(args.config, cfg), "pairs_per_gpu": P, "pairs_total": P_total,
                       "m": m, "n": n, "score_bits": s,
                       "parallelism": f"dp{world} (pair shards)" + (
                           f" on {ngpu} shared GPU(s): code-path check, not a scaling number"
                           if shared else ""),
                       "l2": "inputs 320 MiB > 126 MB L2, plus a 256 MiB L2 flush between steps",
                       "plan": plan},
            "e2e": e2e, "e2e_packed2": e2e_packed2, "filter": filt, "wordwise": wordwise, "roofline": roofline, "cpu_baseline": cpu, "clocks": clocks,
            # ours per step and rank, from the library (fused sweep + extract,
            # or pack + sweep + extract)
            "gpu_launches": plan["kernels"] * args.steps * world, "parity": parity,
            "scores": scores, "w2b_roofline": w2b}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
