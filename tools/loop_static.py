#!/usr/bin/env python
"""Static SASS size of the step kernel's hot loops (pass-1 / pass-2 row loops:
the backward-branch loops with the most HFMA2 / FHADD), opcode histogram.

usage: tools/loop_static.py [LIB.so] [KERNEL_SUBSTR]
"""
import collections
import re
import subprocess
import sys


def sass(lib, kernel):
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    ins, on = [], False
    for line in out.splitlines():
        if "Function :" in line:
            on = kernel in line
            continue
        if on:
            m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
            if m:
                ins.append((int(m.group(1), 16), m.group(2).strip()))
    return ins


def main():
    lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_icpp_fanjzac15_b200/libsharp.so"
    kern = sys.argv[2] if len(sys.argv) > 2 else "step_kernelILb0"
    ins = sass(lib, kern)
    print(f"{kern}: {len(ins)} instructions")
    loops = []
    for a, s in ins:
        m = re.search(r"BRA (?:\S+, )?0x([0-9a-f]+)", s)
        if m and int(m.group(1), 16) < a and "EXIT" not in s:
            t = int(m.group(1), 16)
            body = [x for x in ins if t <= x[0] <= a]
            key = sum(1 for _, b in body if b.split()[0].lstrip("@!P0123456UT ") in () or "FHADD" in b or "HFMA2" in b)
            loops.append((key, t, a, body))
    def hist(body):
        c = collections.Counter()
        for _, b in body:
            op = b.split()[0]
            if op.startswith("@"):
                op = b.split()[1]
            c[op.split(".")[0]] += 1
        return c
    # the innermost loops holding the pass-2 row body (>= 90 FHADD) and the
    # pass-1 row body (>= 20 FHFMA)
    for name, ok in (("pass-2 row loop", lambda c: c["FHADD"] >= 90),
                     ("pass-1 row loop", lambda c: c["PRMT"] >= 20 and c["FHADD"] == 0 and c["HADD2"] + c["HFMA2"] >= 60)):
        cand = [(len(body), t, a, body) for _, t, a, body in loops if ok(hist(body))]
        if not cand:
            continue
        n, t, a, body = min(cand, key=lambda x: x[0])
        c = hist(body)
        print(f"{name} {t:#x}..{a:#x}: {n} instr")
        print("   " + "  ".join(f"{k}:{v}" for k, v in c.most_common(40)))

if __name__ == "__main__":
    main()
