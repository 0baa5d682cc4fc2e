#!/usr/bin/env python3
"""List the backward-branch loops of the kernels matching a regex, with opcode counts.

usage: sass_loops.py <file.o|.so> <kernel-name-regex>
Used to check the sweep's per-step instruction mix.
"""
import re
import subprocess
import sys
from collections import Counter

LINE = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(.*?);")


def main():
    path, pat = sys.argv[1], re.compile(sys.argv[2])
    out = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
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
    for name, ins in funcs.items():
        if not pat.search(name):
            continue
        print(name, "instructions:", len(ins))
        for a, t in ins:
            if "BRA" not in t:
                continue
            m = re.search(r"0x([0-9a-f]+)", t)
            if m and int(m.group(1), 16) < a:
                lo = int(m.group(1), 16)
                loop = [x for b, x in ins if lo <= b <= a]
                c = Counter(re.sub(r"^@!?U?P\w+\s+", "", x).split()[0].split(".")[0] for x in loop)
                print("  loop %#x..%#x: %d instr, %s" % (lo, a, len(loop), ", ".join(
                    "%s=%d" % kv for kv in c.most_common(14))))


if __name__ == "__main__":
    main()
