#!/usr/bin/env python3
"""bench.py -- BPBC Smith-Waterman on B200: GCUPS with bit-exact max local scores.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--impl ours|reference]

One "step" = the whole hot path (W2B transpose of query and target ->
bit-sliced wavefront sweep -> max reduction + B2W untranspose, SURVEY.md
8(a)) over one batch of synthetic pairs already resident in HBM.

Default workload = BASELINE.json configs[2] = C3: 2^22 DNA pairs, m = n =
256, +2/-1/-1, 10-bit slices, "sharded across 1/2/4/8 B200" -- the config
BASELINE's metric ("GCUPS ... at 1/2/4/8 B200") is quoted on.  Under torchrun
(N > 1, one process per GPU) the 2^22 pairs are split by
parallel.shard_range (strong scaling); each rank scores its
shard with no collective on the data path, and the int32 scores are
all-gathered over NCCL once, after the timed region.  At N = 1 the line also
carries a C2 block (configs[1]: 2^20 pairs, m = n = 128, 9 bits).

Prints ONE JSON line on rank 0 (contract in the task statement / DESIGN.md
8): metric, value (GCUPS, all ranks), e2e (the same metric through the
host-buffer C call bpbc_sw_score_batch_host, pinned host inputs, H2D + D2H
inside the timed region, and the measured pinned H2D bandwidth it is bound
by), roofline (the sweep kernel against the measured LOP3 peak), w2b (the
standalone transpose kernel against the measured HBM bandwidth),
cpu_baseline (the oracle on this host's cores: all-core and single-thread
GCUPS, CPU model), parity (N = 1: every pair of the batch checked against
the oracle when that is <= ~40 s of CPU work, else a seeded sample; N > 1:
a 65 536-pair sample of the gathered scores), clocks (nvidia-smi during the
timed region), gpu_launches.

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
DEFAULT_CONFIG = 3
CONSTS = (2, -1, -1)  # match, mismatch, gap (Table II, reading R14)
SM_COUNT = 148
ORACLE_FULL_SECONDS = 60.0  # full oracle parity when the estimate is below this


def workload_name(cid, c):
    name = "paper shape (P:L382)" if cid == 6 else f"C{cid}"
    return (f"{name}: {c['P']} DNA pairs, m={c['m']}, n={c['n']}, "
            f"match/mismatch/gap = +2/-1/-1, {c['s']}-bit score slices, max score only")


def survey_ops_per_word_cell(s):
    """LOP3 form of the circuit, 11s + 2 per 32-cell word."""
    return 11 * s + 2


def measured_lop3_peak():
    """profiles/lop3_peak.json: the LOP3 micro-benchmark (tools/lop3_peak.cu)."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "lop3_peak.json")))
        return float(d["lop3_lane_ops_per_s"]) / 1e12, (
            f"measured: tools/lop3_peak.cu, {d['lanes_per_clk_per_sm_at_max_clock']} LOP3 "
            f"lanes/clk/SM x {d['sms']} SMs at {d['max_clock_mhz']:.0f} MHz "
            "(profiles/lop3_peak.json)")
    except Exception:
        return SM_COUNT * 64 * 1965e6 / 1e12, ("fallback: 148 SMs x 64 LOP3 lanes/clk x 1965 MHz "
                                              "(B300_MICROARCH alu rt = 2 per SMSP)")


def hbm_peak():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]), \
            "MEASURED_PEAKS.json hbm_gbs"
    except Exception:
        return 6460.5, "fallback 6460.5 GB/s (MEASURED_PEAKS.json unreadable)"


def ncu_evidence(key):
    """Committed ncu numbers of the sweep kernel for a config (profiles/ncu_sweep.json,
    written by tools/ncu_summary.py json): DRAM bytes per launch and alu-pipe %."""
    try:
        return json.load(open(os.path.join(ROOT, "profiles", "ncu_sweep.json"))).get(key)
    except Exception:
        return None


def cpu_model():
    try:
        for ln in subprocess.run(["lscpu"], capture_output=True, text=True).stdout.splitlines():
            if ln.startswith("Model name"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


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


def oracle_rate(q, t, s, threads):
    """Oracle pairs/s on a warm library with enough pairs per thread."""
    import oracle
    cells = q.shape[1] * t.shape[1]
    # ~0.2 s per thread of work, at least one pair per thread
    cal = min(q.shape[0], max(threads, min(max(64 * threads, 2048), int(2e8 * threads / cells))))
    oracle.sw_batch(q[:threads], t[:threads], *CONSTS, score_bits=s, threads=threads)
    t0 = time.perf_counter()
    oracle.sw_batch(q[:cal], t[:cal], *CONSTS, score_bits=s, threads=threads)
    return cal / max(time.perf_counter() - t0, 1e-6)


def parity_and_cpu_baseline(q, t, got, cfg, label, sample_pairs=None):
    """The oracle on this host's cores checks the GPU scores (every pair when
    that fits ORACLE_FULL_SECONDS, else a seeded sample) and the same run is
    the all-core cpu_baseline; a ~3 s single-thread run gives the paper's own
    CPU methodology (sequential)."""
    import oracle
    threads = os.cpu_count() or 1
    P, m = q.shape
    n = t.shape[1]
    s = cfg["s"]
    rate = oracle_rate(q, t, s, threads)
    if sample_pairs is None and P / rate <= ORACLE_FULL_SECONDS:
        idx = None
        what = f"all {P} pairs"
    else:
        k = min(P, sample_pairs or max(4096, int(rate * ORACLE_FULL_SECONDS / 2)))
        rng = np.random.default_rng(cfg["P"] + m + n)
        idx = np.sort(rng.choice(P, size=k, replace=False)) if k < P else None
        what = f"a seeded sample of {k} of the {P} pairs" if idx is not None else f"all {P} pairs"
    qq, tt = (q, t) if idx is None else (q[idx], t[idx])
    gg = got if idx is None else got[idx]
    t0 = time.perf_counter()
    want = oracle.sw_batch(qq, tt, *CONSTS, score_bits=s, threads=threads)
    dt = time.perf_counter() - t0
    mism = int((gg != want).sum())
    # single thread (the paper's CPU methodology)
    r1 = oracle_rate(q, t, s, 1)
    k1 = int(min(P, max(8, r1 * 3.0)))
    t1 = time.perf_counter()
    oracle.sw_batch(q[:k1], t[:k1], *CONSTS, score_bits=s, threads=1)
    d1 = time.perf_counter() - t1
    cells = qq.shape[0] * m * n
    parity = {"pairs_checked": int(qq.shape[0]), "mismatches": mism, "scope": what,
              "what": f"GPU scores of {label} vs the CPU oracle (oracle/sw_oracle.c), bit-exact"}
    cpu = {"value": round(cells / dt / 1e9, 4), "unit": "GCUPS", "cores": threads,
           "kind": "oracle",
           "single_thread_gcups": round(k1 * m * n / d1 / 1e9, 4),
           "cpu_model": cpu_model(),
           "sample": f"{what} of {label} (m={m}, n={n}), {dt:.1f} s on {threads} threads, "
                     f"scalar int32 DP; single thread: first {k1} pairs, {d1:.1f} s"}
    return parity, cpu


def gathered_sample_index(P_total, m, k=65536):
    """N > 1 parity: the seeded sample of global pair indices rank 0 checks."""
    k = min(P_total, k)
    rng = np.random.default_rng(P_total + m)
    return np.sort(rng.choice(P_total, size=k, replace=False))


def regen_pairs(seed, idx, m, n):
    """Pairs idx (sorted global indices) of the batch: every rank generated
    its shard with p_offset = its first global pair index, so pair p of the
    gathered batch is gen(p_offset=p) (counter-based generator, synth/)."""
    import synth
    qs = np.empty((idx.size, m), dtype=np.uint8)
    ts = np.empty((idx.size, n), dtype=np.uint8)
    runs = np.split(idx, np.nonzero(np.diff(idx) != 1)[0] + 1) if idx.size else []
    j = 0
    for r in runs:
        a, b = int(r[0]), int(r[-1]) + 1
        qa, ta = synth.gen_pairs(seed, b - a, m, n, p_offset=a)
        qs[j:j + b - a], ts[j:j + b - a] = qa, ta
        j += b - a
    return qs, ts


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
    cal = int(min(cfg["P"], max(64 * threads, 4096)))
    q, t = synth.gen_pairs(seed, cal, m, n)
    rate = oracle_rate(q, t, cfg["s"], threads)
    # size one step so the whole run stays within ~1-2 minutes
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
                             "kind": "oracle", "cpu_model": cpu_model(),
                             "sample": f"{per_step} pairs of C{cfg['id']} per step"},
            "e2e": {"value": round(v, 4), "unit": "GCUPS", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def time_device_steps(fn, steps, warmup, flush):
    """CUDA-event time of `steps` calls of fn (L2 flushed between them)."""
    import torch
    for _ in range(warmup):
        fn()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    torch.cuda.synchronize()
    for k in range(steps):
        flush.zero_()
        starts[k].record()
        fn()
        ends[k].record()
    torch.cuda.synchronize()
    return sum(a.elapsed_time(b) for a, b in zip(starts, ends))


def sweep_roofline(plan, phases, P, m, n, s, key):
    """The dominant kernel (the sweep) against the measured LOP3 peak."""
    calls = max(1, phases["calls"])
    sweep_ms = phases["swa_ms"] / calls
    word_cells = (P + 31) // 32 * m * n
    peak, peak_src = measured_lop3_peak()
    ops = plan["ops_per_word_cell"]
    achieved = ops * word_cells / (sweep_ms / 1e3) / 1e12
    achieved_survey = survey_ops_per_word_cell(s) * word_cells / (sweep_ms / 1e3) / 1e12
    ev = ncu_evidence(key) or {}
    kernel = "sw_sweep_wrap_kernel" if plan.get("wrap") else (
        "sw_sweep_kernel" if plan.get("fused") else "sw_sweep_mw_kernel / striped")
    return {"bound": "alu", "achieved": round(achieved, 3), "peak": round(peak, 3),
            "unit": "Tops/s (LOP3 lane-ops)", "frac": round(achieved / peak, 4),
            "traffic": ev.get("dram_bytes"),
            "frac_survey_11s_plus_2": round(achieved_survey / peak, 4),
            "alu_pipe_pct_ncu": ev.get("alu_pipe_pct"),
            "ncu_source": ev.get("source"),
            "kernel": kernel, "kernel_ms_per_launch": round(sweep_ms, 4),
            "alg_ops_per_word_cell": ops,
            "alg_ops_per_word_cell_survey": survey_ops_per_word_cell(s),
            "word_cells_per_launch": word_cells, "peak_basis": peak_src,
            "phase_ms_per_step": {k: round(v / calls, 4) for k, v in phases.items()
                                  if k.endswith("_ms")}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=DEFAULT_CONFIG, choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-extra", action="store_true",
                    help="skip the C2 block, filter, wordwise and W2B lines")
    ap.add_argument("--no-filter", action="store_true", help="(alias of --no-extra)")
    ap.add_argument("--score-bits", type=int, default=None)
    ap.add_argument("--m", type=int, default=None, help="override the query length")
    ap.add_argument("--n", type=int, default=None, help="override the target length")
    ap.add_argument("--pairs", type=int, default=None, help="override the pair count")
    ap.add_argument("--filter-threshold", type=int, default=None,
                    help="tau of the threshold-filter line (default 0.9 * min(m, n))")
    args = ap.parse_args()
    args.no_extra = args.no_extra or args.no_filter
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
    from paper_conf_ipps_nishimurabin17_b200 import parallel

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
    ws = torch.empty(bpbc.workspace_bytes_for(P, m, n, *CONSTS, score_bits=s, device=local),
                     dtype=torch.uint8, device=dev)
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
    roofline = sweep_roofline(plan, phases, P, m, n, s, f"C{args.config}")

    # ---------------- extras on this rank's resident batch (rank-local numbers)
    filt = wordwise = w2b = c2 = None
    if not args.no_extra:
        tau = args.filter_threshold if args.filter_threshold is not None else int(0.9 * min(m, n))
        fws = torch.empty(bpbc.workspace_bytes_for(P, m, n, *CONSTS, score_bits=s, filter=True,
                                                   device=local), dtype=torch.uint8, device=dev)
        fk = max(3, min(args.steps, 10))
        f_ms = time_device_steps(
            lambda: bpbc.filter_batch(dq, dt, tau, *CONSTS, score_bits=s, workspace=fws),
            fk, args.warmup, flush)
        _, cnt, _ = bpbc.filter_batch(dq, dt, tau, *CONSTS, score_bits=s, workspace=fws)
        filt = {"value": round(P * m * n * fk / (f_ms / 1e3) / 1e9, 2), "unit": "GCUPS",
                "threshold": tau, "flagged_pairs_rank0": int(cnt.item()),
                "ms_per_step": round(f_ms / fk, 4),
                "what": "bpbc_sw_filter_batch: pairs with max score > threshold, mask + "
                        "ascending indices (P:L231)"}
        del fws
        if min(m, n) <= 256:
            wout = torch.empty(P, dtype=torch.int32, device=dev)
            wk = max(3, min(args.steps, 10))
            w_ms = time_device_steps(lambda: bpbc.score_batch_wordwise(dq, dt, *CONSTS, out=wout),
                                     wk, args.warmup, flush)
            wv = P * m * n * wk / (w_ms / 1e3) / 1e9
            agree = bool(torch.equal(torch.clamp(wout, max=(1 << s) - 1), out))
            wordwise = {"value": round(wv, 2), "unit": "GCUPS", "ms_per_step": round(w_ms / wk, 4),
                        "bitwise_over_wordwise": round(gcups / world / wv, 3) if wv else None,
                        "agrees_with_bitwise": agree,
                        "what": "bpbc_sw_score_batch_wordwise: ordinary-integer DP, 16-bit SIMD, "
                                "2 pairs per warp register (the paper's GPU wordwise row, P:L407)"}
            del wout
        # W2B (a1+a2) alone: the standalone transpose kernel (bpbc_sw_pack) on
        # the same resident inputs, against the measured HBM bandwidth; the
        # hot path runs it fused into the sweep
        hbm, hbm_src = hbm_peak()
        G = (P + 31) // 32
        pq = torch.empty((G, m, 2), dtype=torch.int32, device=dev)
        pt = torch.empty((G, n, 2), dtype=torch.int32, device=dev)
        pk = max(3, min(args.steps, 10))
        p_ms = time_device_steps(lambda: (bpbc.pack(dq, out=pq), bpbc.pack(dt, out=pt)),
                                 pk, args.warmup, flush)
        nbytes = P * (m + n) + 8 * G * (m + n)  # u8 codes read + uint2 planes written
        gbs = nbytes / (p_ms / pk / 1e3) / 1e9
        w2b = {"bound": "hbm", "kernel": "pack_kernel (bpbc_sw_pack, query + target)",
               "achieved": round(gbs, 1), "peak": hbm, "unit": "GB/s",
               "frac": round(gbs / hbm, 4), "bytes_per_step": nbytes,
               "ms_per_step": round(p_ms / pk, 4), "peak_source": hbm_src,
               "ncu": ncu_evidence(f"W2B_C{args.config}")}
        del pq, pt

    # ---------------- end to end through the host-buffer C call
    e2e = e2e_packed2 = None
    if not args.no_e2e:
        # pinned H2D bandwidth of the same bytes (the bound of the u8 path)
        hbuf = hq.view(-1)[: min(hq.numel(), 1 << 30)]
        dbuf = torch.empty_like(hbuf, device=dev)
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for _ in range(2):
            dbuf.copy_(hbuf, non_blocking=True)
        torch.cuda.synchronize()
        ev0.record()
        for _ in range(3):
            dbuf.copy_(hbuf, non_blocking=True)
        ev1.record()
        torch.cuda.synchronize()
        h2d_gbs = 3 * hbuf.numel() / (ev0.elapsed_time(ev1) / 1e3) / 1e9
        del dbuf
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
        e2e_host_ok = bool((hout.numpy() == out.cpu().numpy()).all())
        bound_gcups = P_total * m * n / (P_total * (m + n) / (h2d_gbs * 1e9)) / 1e9
        e2e = {"value": round(P_total * m * n * ksteps / el / 1e9, 2), "unit": "GCUPS",
               "h2d_bytes_per_step": P_total * (m + n), "d2h_bytes_per_step": P_total * 4,
               "steps": ksteps, "equals_device_scores": e2e_host_ok,
               "pinned_h2d_gbs": round(h2d_gbs, 2),
               "h2d_bound_gcups": round(bound_gcups, 1),
               "frac_of_min_device_h2d_bound": round(
                   P_total * m * n * ksteps / el / 1e9 / min(gcups, bound_gcups), 4),
               "timing": "host wall clock around the blocking C call bpbc_sw_score_batch_host "
                         "(pinned host buffers, 1 byte per base; 3 slots / 3 streams)"}
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
        v2 = P_total * m * n * ksteps / el2 / 1e9
        e2e_packed2 = {"value": round(v2, 2), "unit": "GCUPS",
                       "h2d_bytes_per_step": P_total * ((m + 3) // 4 + (n + 3) // 4),
                       "d2h_bytes_per_step": P_total * 4, "steps": ksteps,
                       "frac_of_device": round(v2 / gcups, 4),
                       "timing": "host wall clock around bpbc_sw_score_batch_host_packed2 "
                                 "(pinned, 2-bit packed bases)"}
        del hq2, ht2

    # ---------------- C2 block (N = 1, default config): BASELINE configs[1]
    if not args.no_extra and world == 1 and args.config == DEFAULT_CONFIG and not (
            args.m or args.n or args.pairs or args.score_bits):
        c2cfg = dict(CONFIGS[2], id=2)
        P2, m2, n2, s2 = c2cfg["P"], c2cfg["m"], c2cfg["n"], c2cfg["s"]
        q2, t2 = synth.gen_pairs(synth.seed_for_config(2), P2, m2, n2)
        dq2, dt2 = torch.from_numpy(q2).to(dev), torch.from_numpy(t2).to(dev)
        out2 = torch.empty(P2, dtype=torch.int32, device=dev)
        ws2 = torch.empty(bpbc.workspace_bytes_for(P2, m2, n2, *CONSTS, score_bits=s2,
                                                   device=local), dtype=torch.uint8, device=dev)
        bpbc.profile(True, local)
        c2_ms = time_device_steps(lambda: bpbc.score_batch(dq2, dt2, *CONSTS, score_bits=s2,
                                                           out=out2, workspace=ws2),
                                  args.steps, args.warmup, flush)
        ph2 = bpbc.profile_read(local)
        bpbc.profile(False, local)
        plan2 = bpbc.last_plan(local)
        g2 = out2.cpu().numpy()
        par2, _ = (parity_and_cpu_baseline(q2, t2, g2, c2cfg, "C2", sample_pairs=65536)
                   if not args.no_cpu_baseline else (None, None))
        c2 = {"value": round(P2 * m2 * n2 * args.steps / (c2_ms / 1e3) / 1e9, 2),
              "unit": "GCUPS", "ms_per_step": round(c2_ms / args.steps, 4),
              "workload": workload_name(2, c2cfg), "plan": plan2,
              "roofline": sweep_roofline(plan2, ph2, P2, m2, n2, s2, "C2"), "parity": par2}
        del dq2, dt2, out2, ws2

    # ---------------- result gather (outside the timed region)
    if world > 1:  # rank r holds the pairs of shard_range(P_total, world, r)
        if cfg["scaling"] == "strong":
            full = parallel.gather_scores(out.to(cdev), P_total)
        else:  # weak: equal shards of cfg["P"] pairs, rank-major
            parts = [torch.empty(P, dtype=torch.int32, device=cdev) for _ in range(world)]
            dist.all_gather(parts, out.to(cdev))
            full = torch.cat(parts)
        got_all = full.cpu().numpy()
    else:
        got_all = out.cpu().numpy()
    if rank != 0:
        dist.destroy_process_group()
        return

    cpu = parity = None
    if not args.no_cpu_baseline:
        if world == 1:
            parity, cpu = parity_and_cpu_baseline(hq.numpy(), ht.numpy(), got_all, cfg,
                                                  f"C{args.config}")
        else:
            # rank 0 regenerates a 65 536-pair sample of the WHOLE gathered
            # batch (every rank's shard) from the counter-based generator
            idx = gathered_sample_index(P_total, m)
            qs, ts = regen_pairs(seed, idx, m, n)
            k = idx.size
            parity, cpu = parity_and_cpu_baseline(qs, ts, got_all[idx], cfg,
                                                  f"C{args.config} (gathered over {world} ranks)",
                                                  sample_pairs=k)
    # score distribution of the batch (C5: the share capped at 2^s - 1, R3)
    scores = {"mean": round(float(got_all.mean()), 3), "max": int(got_all.max()),
              "saturated_frac": round(float((got_all == (1 << s) - 1).mean()), 6)}
    shards = [list(parallel.shard_range(P_total, world, r)) for r in range(world)] \
        if cfg["scaling"] == "strong" else [[r * cfg["P"], (r + 1) * cfg["P"]] for r in range(world)]

    line = {"metric": METRIC, "value": round(gcups, 2), "unit": "GCUPS", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(t_ms / args.steps, 4), "higher_is_better": True,
            "scaling": cfg["scaling"], "vs_baseline": None,
            "dtype": "u32 bit-sliced (s-bit scores)",
            "data": "synthetic (seeded i.i.d. uniform DNA, SplitMix64)",
            "config": {"workload": workload_name(args.config, cfg), "pairs_total": P_total,
                       "pairs_per_gpu": P, "rank_shards": shards,
                       "m": m, "n": n, "score_bits": s,
                       "parallelism": f"dp{world} (pair shards, no data-path collective; NCCL "
                                      "all-gather of the int32 scores after the timed region)"
                                      + (f" on {ngpu} shared GPU(s): code-path check, not a "
                                         "scaling number" if shared else ""),
                       "l2": "inputs > 126 MB L2, plus a 256 MiB L2 flush between steps",
                       "plan": plan},
            "e2e": e2e, "e2e_packed2": e2e_packed2, "roofline": roofline, "w2b": w2b,
            "cpu_baseline": cpu, "parity": parity, "clocks": clocks,
            # ours per step and rank, from the library (fused sweep + extract,
            # or pack + sweep + extract)
            "gpu_launches": plan["kernels"] * args.steps * world,
            "scores": scores, "c2": c2, "filter": filt, "wordwise": wordwise}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
