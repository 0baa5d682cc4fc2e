#!/usr/bin/env python3
"""SASS evidence for the headline sweep kernels (north_star: "has its SASS
inspected"): for each kernel, the instruction mix of its hot loops and the
LOP3 count per word-cell of the switch-free loop against the hand count of
the circuit the plan evaluates (the paper's op count is
Theorem 6).

usage: python tools/sass_report.py [--build build/csrc] [--json]

The "switch-free loop" is the straight-line two-step block of the hot loop
without the group-switch code (the switch copy runs only in switch windows).
One word-cell = one 32-bit word of one DP cell = 32 cells.  A loop
iteration runs two wavefront steps of R rows per lane, i.e. 2 R word-cells
per thread, so LOP3 per word-cell = LOP3 in the loop / (2 R).
"""
import argparse
import json
import os
import re
import subprocess
from collections import Counter

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LINE = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(.*?);")

# (label, object width, kernel-name pattern, rows per lane R, hand count per word-cell)
# hand counts: exact circuit 10 S, saturating 11 S + 2 (compile-time (+2,-1,-1))
HEADLINE = [
    ("C1/C4 (m=64: s=8, R=4, L=16)", 8, r"sw_sweep_kernelILi8ELi4ELi16ELi0ELb0ENS_4KFixILi2ELi1ELi1E", 4, 80),
    ("C2 (m=128: s=9, R=4, L=32)", 9, r"sw_sweep_kernelILi9ELi4ELi32ELi0ELb0ENS_4KFixILi2ELi1ELi1E", 4, 90),
    ("C3 (m=256: s=10, R=8, L=32)", 10, r"sw_sweep_kernelILi10ELi8ELi32ELi0ELb0ENS_4KFixILi2ELi1ELi1E", 8, 100),
    ("C5 m=32 (s=7, R=2, L=16)", 7, r"sw_sweep_kernelILi7ELi2ELi16ELi0ELb0ENS_4KFixILi2ELi1ELi1E", 2, 70),
    ("C5 m=512 (s=11, multi-warp R=4, W=4)", 11, r"sw_sweep_mw_kernelILi11ELi4ELi4ELi0ENS_4KFixILi2ELi1ELi1E", 4, 110),
    ("paper shape (m=128: s=9, wrap-around, R=4)", 9, r"sw_sweep_wrap_kernelILi9ELi4ELi0ELb0ENS_4KFixILi2ELi1ELi1E", 4, 90),
    ("C2 saturating s=9 (11s+2 circuit)", 9, r"sw_sweep_kernelILi9ELi4ELi32ELi1ELb0ENS_4KFixILi2ELi1ELi1E", 4, 101),
]


def kernel_symbols(obj):
    """Mangled names of the device kernels in obj (from the host stubs)."""
    out = subprocess.run(["nm", obj], capture_output=True, text=True).stdout
    return sorted({ln.split()[-1] for ln in out.splitlines() if "sw_sweep" in ln and "Sweep" in ln})


def sass_functions(obj, names=None):
    cmd = ["cuobjdump", "-sass", obj]
    if names:
        cmd[2:2] = ["-fun", ",".join(names)]
    out = subprocess.run(cmd, capture_output=True, text=True).stdout
    funcs, cur = {}, None
    for ln in out.splitlines():
        m = re.search(r"Function : (\S+)", ln)
        if m:
            cur = m.group(1)
            funcs[cur] = []
            continue
        mm = LINE.search(ln)
        if mm and cur:
            funcs[cur].append((int(mm.group(1), 16), mm.group(2).strip()))
    return funcs


def opcode(text):
    return re.sub(r"^@!?U?P\w+\s+", "", text).split()[0].split(".")[0]


def loops(ins):
    """Innermost backward-branch loops: (lo, hi, Counter of opcodes)."""
    found = []
    for a, t in ins:
        if "BRA" not in t:
            continue
        m = re.search(r"0x([0-9a-f]+)", t)
        if m and int(m.group(1), 16) < a:
            lo = int(m.group(1), 16)
            body = [opcode(x) for b, x in ins if lo <= b <= a]
            found.append((lo, a, Counter(body)))
    # innermost: loops that contain no other loop
    inner = [l for l in found if not any(o is not l and l[0] <= o[0] and o[1] <= l[1]
                                         and (o[0], o[1]) != (l[0], l[1]) for o in found)]
    return inner


def basic_blocks(ins, lo, hi):
    """Split a loop body into straight-line blocks at branches and at the
    targets of branches inside it: [(start, end, Counter of opcodes)]."""
    targets = set()
    for a, t in ins:
        m = re.search(r"BRA(?:\.\w+)*\s.*?0x([0-9a-f]+)", t)
        if m and lo <= int(m.group(1), 16) <= hi:
            targets.add(int(m.group(1), 16))
    out, cur, start = [], Counter(), None
    for a, t in ins:
        if a in targets and cur:
            out.append((start, prev, cur))
            cur, start = Counter(), None
        if start is None:
            start = a
        cur[opcode(t)] += 1
        prev = a
        if "BRA" in t:
            out.append((start, a, cur))
            cur, start = Counter(), None
    if cur:
        out.append((start, prev, cur))
    return out


def report(build):
    rows = []
    for label, width, pat, R, hand in HEADLINE:
        obj = os.path.join(build, f"sweep_s{width}_m0.o")
        syms = [f for f in kernel_symbols(obj) if re.search(pat, f)]
        funcs = sass_functions(obj, syms[:1]) if syms else {}
        name = next((f for f in funcs if re.search(pat, f)), None)
        if name is None:
            rows.append({"kernel": label, "error": f"{pat} not found in {obj}"})
            continue
        inner = [l for l in loops(funcs[name]) if l[2]["LOP3"] > 100]
        # straight-line blocks of the hot loops (split at branches and branch
        # targets): the switch-free two-step body = the big block with the
        # fewest non-LOP3 instructions
        blocks = []
        for lo, hi, _ in inner:
            blocks += basic_blocks([(a_, t) for a_, t in funcs[name] if lo <= a_ <= hi], lo, hi)
        # a candidate holds two whole steps (>= 90 % of the hand count's LOP3);
        # loops whose steps contain a divergent switch branch (R = 8, the
        # multi-warp kernel) are taken whole
        need = 0.9 * 2 * R * hand
        cands = [b_ for b_ in blocks if b_[2]["LOP3"] >= need] or \
                [l for l in inner if l[2]["LOP3"] >= need]
        blocks = [b_ for b_ in blocks if b_[2]["LOP3"] > 100]
        best = min(cands, key=lambda l: sum(l[2].values()) - l[2]["LOP3"])
        total = sum(best[2].values())
        lop3 = best[2]["LOP3"]
        rows.append({"kernel": label, "symbol_pattern": pat, "loop": f"{best[0]:#x}..{best[1]:#x}",
                     "instructions": total, "lop3": lop3, "rows_per_lane": R,
                     "lop3_per_word_cell": lop3 / (2 * R), "hand_count": hand,
                     "other": {k: v for k, v in best[2].most_common() if k != "LOP3"},
                     "loops": [{"range": f"{l[0]:#x}..{l[1]:#x}", "instructions": sum(l[2].values()),
                                "lop3": l[2]["LOP3"]} for l in inner],
                     "blocks": [{"range": f"{b_[0]:#x}..{b_[1]:#x}", "instructions": sum(b_[2].values()),
                                 "lop3": b_[2]["LOP3"]} for b_ in blocks]})
    return rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--build", default=os.path.join(ROOT, "build", "csrc"))
    ap.add_argument("--json", action="store_true")
    a = ap.parse_args()
    rows = report(a.build)
    if a.json:
        print(json.dumps(rows, indent=1))
        return
    print("| kernel | switch-free block | instr / 2 steps | LOP3 / 2 steps | LOP3 per word-cell | hand count | other opcodes |")
    print("|---|---|---|---|---|---|---|")
    for r in rows:
        if "error" in r:
            print(f"| {r['kernel']} | {r['error']} | | | | | |")
            continue
        other = ", ".join(f"{k} {v}" for k, v in r["other"].items())
        print(f"| {r['kernel']} | {r['loop']} | {r['instructions']} | {r['lop3']} | "
              f"{r['lop3_per_word_cell']:.2f} | {r['hand_count']} | {other} |")


if __name__ == "__main__":
    main()
