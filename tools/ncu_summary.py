#!/usr/bin/env python3
"""Summarise ncu captures for profiles/ (run here, no GPU needed).

usage:
  ncu_summary.py report <file.ncu-rep> [...]   key metrics of every captured kernel
  ncu_summary.py launches <launches.csv>       per-kernel launch count, mean time, share of the step
  ncu_summary.py json <file.ncu-rep> <KEY> [kernel-regex]
                                               record the first matching kernel's DRAM bytes and
                                               alu-pipe % under KEY in profiles/ncu_sweep.json
                                               (read by bench.py's roofline)

The metric list is the one DESIGN.md cites: duration, DRAM bytes (the
roofline `traffic`), alu / fma / lsu pipe utilisation, issue activity,
occupancy, registers and the top stall reasons.
"""
import csv
import io
import re
import subprocess
import sys
from collections import OrderedDict, defaultdict

KEYS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "launch__occupancy_limit_registers",
    "sm__cycles_active.avg",
    "inst_executed",
]
STALL = re.compile(r"smsp__average_warps_issue_stalled_(\w+)_per_issue_active\.ratio")


def raw_csv(path):
    """--page raw --csv of a report, or the exported text itself (.csv)."""
    if path.endswith(".csv"):
        return open(path).read()
    return subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                          text=True).stdout


def report(path):
    raw = raw_csv(path)
    rows = list(csv.reader(io.StringIO(raw)))
    if len(rows) < 3:
        print(f"{path}: no data")
        return
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        name = d.get("Kernel Name", "?")
        print(f"== {path}: {name[:140]}")
        for k in KEYS:
            if k in d:
                print(f"  {k:<62} {d[k]:>16} {u.get(k, '')}")
        stalls = []
        for k, v in d.items():
            m = STALL.match(k)
            if m:
                try:
                    stalls.append((float(v), m.group(1)))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        print("  top stalls (warps per issue): " +
              ", ".join(f"{n}={v:.3f}" for v, n in stalls[:6]))


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = OrderedDict()
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        name = re.sub(r"\(.*", "", r[ki])
        agg.setdefault(name, []).append(float(r[vi].replace(",", "")))
    total = sum(sum(v) for v in agg.values())
    print(f"{'kernel':<70} {'launches':>8} {'mean_us':>10} {'share':>7}")
    for k, v in agg.items():
        print(f"{k[:70]:<70} {len(v):>8} {sum(v) / len(v) / 1e3:>10.2f} {sum(v) / total:>7.1%}")


def record(path, key, pattern="sw_sweep"):
    import json
    import os
    raw = raw_csv(path)
    rows = list(csv.reader(io.StringIO(raw)))
    hdr = rows[0]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        if not re.search(pattern, d.get("Kernel Name", "")):
            continue
        num = lambda k: float(d[k].replace(",", ""))
        # ncu reports bytes in the unit of row 1 (Mbyte / Gbyte / byte)
        units = dict(zip(hdr, rows[1]))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        dram = sum(num(k) * scale.get(units[k], 1) for k in ("dram__bytes_read.sum",
                                                              "dram__bytes_write.sum"))
        entry = {"dram_bytes": int(dram),
                 "alu_pipe_pct": round(num("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"), 2),
                 "duration_ms": round(num("gpu__time_duration.sum") *
                                      {"us": 1e-3, "usecond": 1e-3, "ms": 1, "msecond": 1, "ns": 1e-6, "nsecond": 1e-6}.get(
                                          units["gpu__time_duration.sum"], 1), 4),
                 "kernel": re.sub(r"\(.*", "", d["Kernel Name"])[:120],
                 "source": os.path.basename(path) + " (ncu --set full, one launch)"}
        out = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                           "ncu_sweep.json")
        allj = json.load(open(out)) if os.path.exists(out) else {}
        allj[key] = entry
        json.dump(allj, open(out, "w"), indent=1, sort_keys=True)
        print(key, entry)
        return
    print(f"{path}: no kernel matches {pattern}")


def main():
    if len(sys.argv) < 3:
        print(__doc__)
        sys.exit(2)
    if sys.argv[1] == "json":
        record(sys.argv[2], sys.argv[3], *(sys.argv[4:5] or []))
        return
    if sys.argv[1] == "report":
        for p in sys.argv[2:]:
            report(p)
    else:
        launches(sys.argv[2])


if __name__ == "__main__":
    main()
