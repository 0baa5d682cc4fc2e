#!/usr/bin/env python3
"""Executed-instruction mix of one kernel from an ncu source export
(ncu -i REP --page source --csv --print-source sass > FILE.csv).

usage: ncu_opmix.py FILE.csv [word_cells]
Prints warp-level instructions executed per opcode (and per word-cell when
the launch's word-cell count is given), split into the pipes the sweep
cares about, plus the share of stall samples per opcode.
"""
import csv
import gzip
import re
import sys
from collections import Counter

ALU = {"LOP3", "ISETP", "SEL", "SHF", "IADD3", "PLOP3", "LEA", "FLO", "POPC", "BMSK", "PRMT",
       "VIADD", "VIMNMX", "IMNMX", "LOP", "SGXT", "CSETP", "P2R", "R2P"}


def main():
    rows = list(csv.reader(gzip.open(sys.argv[1], "rt") if sys.argv[1].endswith(".gz") else open(sys.argv[1])))
    h = rows[1]
    ie = h.index("Instructions Executed")
    src = h.index("Source")
    smp = h.index("Warp Stall Sampling (All Samples)")
    ops, samples = Counter(), Counter()
    for r in rows[2:]:
        op = re.sub(r"^@!?U?P\w+\s+", "", r[src].strip()).split()[0].split(".")[0] if r[src].strip() else "?"
        ops[op] += int(r[ie] or 0)
        samples[op] += int(r[smp] or 0)
    tot = sum(ops.values())
    wc = float(sys.argv[2]) if len(sys.argv) > 2 else None
    alu = sum(v for k, v in ops.items() if k in ALU)
    ts = sum(samples.values()) or 1
    print(f"total warp instructions {tot}, alu-pipe class {alu} ({100 * alu / tot:.1f} %)")
    if wc:
        print(f"per word-cell: total {tot * 32 / wc:.2f} thread-ops... (warp instr x 32 / word-cells)")
    for k, v in ops.most_common(25):
        extra = f"  {v * 32 / wc:8.2f} /word-cell" if wc else ""
        print(f"  {k:10s} {v:14d} {100 * v / tot:6.2f} %  stall-samples {100 * samples[k] / ts:5.1f} %{extra}")


if __name__ == "__main__":
    main()
