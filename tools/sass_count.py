#!/usr/bin/env python3
"""Count SASS opcodes of a kernel, overall and inside its innermost hot loop.

usage: sass_count.py <file.o|.so|.cubin> [kernel-name-regex]

The hot loop is taken as the largest span [target, BRA] of a backward branch.
Used to check the LOP3 count per word-cell of the sweep kernel.
"""
import re
import subprocess
import sys
from collections import Counter

LINE = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.[A-Z0-9_.]*)?\s*([^;]*);")


def kernels(path):
    out = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
    cur, body = None, []
    res = {}
    for ln in out.splitlines():
        m = re.search(r"Function : (\S+)", ln)
        if m:
            if cur:
                res[cur] = body
            cur, body = m.group(1), []
            continue
        mm = LINE.search(ln)
        if mm and cur:
            body.append((int(mm.group(1), 16), mm.group(3), mm.group(4) or "", mm.group(5)))
    if cur:
        res[cur] = body
    return res


def hot_loop(body):
    best = None
    for addr, op, mod, args in body:
        if op == "BRA":
            m = re.search(r"0x([0-9a-f]+)", args)
            if m:
                tgt = int(m.group(1), 16)
                if tgt < addr and (best is None or addr - tgt > best[1] - best[0]):
                    best = (tgt, addr)
    if not best:
        return []
    return [x for x in body if best[0] <= x[0] <= best[1]]


def main():
    path = sys.argv[1]
    pat = re.compile(sys.argv[2]) if len(sys.argv) > 2 else None
    for name, body in kernels(path).items():
        if pat and not pat.search(name):
            continue
        loop = hot_loop(body)
        c = Counter(op for _, op, _, _ in loop)
        print(name)
        print("  total instr %d, hot-loop instr %d" % (len(body), len(loop)))
        print("  loop:", ", ".join("%s=%d" % kv for kv in c.most_common()))


if __name__ == "__main__":
    main()
