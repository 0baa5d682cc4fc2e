#!/usr/bin/env python3
"""Split an ncu source-page export (--page source --csv --print-source sass) of one
kernel into code regions (the backward-branch loops found by sass_loops.py, given
as hex offset ranges) and print executed instructions and stall samples per region.

usage: ncu_regions.py <source.csv> name=0xa-0xb [name=0xc-0xd ...]
Used for the sweep kernel's fast / switch / per-phase split.
"""
import csv
import gzip
import sys
from collections import Counter, defaultdict


def main():
    rows = list(csv.reader(gzip.open(sys.argv[1], "rt") if sys.argv[1].endswith(".gz") else open(sys.argv[1])))
    ranges = {}
    for arg in sys.argv[2:]:
        k, v = arg.split("=")
        a, b = v.split("-")
        ranges[k] = (int(a, 16), int(b, 16))
    h = rows[1]
    ia, isrc, iadr = h.index("Instructions Executed"), h.index("Source"), h.index("Address")
    iss = h.index("Warp Stall Sampling (All Samples)")
    stalls = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
    base = int(rows[2][iadr], 16)
    inst, samp, st, lop = Counter(), Counter(), defaultdict(Counter), Counter()
    for r in rows[2:]:
        off = int(r[iadr], 16) - base
        reg = next((k for k, (a, b) in ranges.items() if a <= off <= b), "other")
        n = int(r[ia] or 0)
        inst[reg] += n
        if "LOP3" in r[isrc]:
            lop[reg] += n
        samp[reg] += int(r[iss] or 0)
        for c in stalls:
            st[reg][c[6:]] += int(r[h.index(c)] or 0)
    tot = sum(samp.values())
    for reg in list(ranges) + ["other"]:
        print(f"{reg:8s} inst {inst[reg]:12d} lop3 {lop[reg]:12d} samples {samp[reg]:7d} "
              f"({100 * samp[reg] / max(tot, 1):5.1f}%)  samples/Mlop3 {samp[reg] / max(lop[reg], 1) * 1e6:7.1f}")
        print("         ", {k: v for k, v in st[reg].most_common(8) if v})


if __name__ == "__main__":
    main()
