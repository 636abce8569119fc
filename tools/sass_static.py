#!/usr/bin/env python
"""Static SASS opcode histogram of step_kernel in libsharp.so (or a diff of two).

usage: tools/sass_static.py [LIB.so] [OTHER.so]
"""
import collections
import re
import subprocess
import sys


def hist(lib, kernel="step_kernel"):
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    body, on = [], False
    for line in out.splitlines():
        if "Function :" in line:
            on = kernel in line
            continue
        if on:
            m = re.match(r"\s*/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)", line)
            if m:
                body.append(m.group(2))
    c = collections.Counter(op.split(".")[0] for op in body)
    return len(body), c


def main():
    a = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_icpp_fanjzac15_b200/libsharp.so"
    n, c = hist(a)
    if len(sys.argv) > 2:
        n2, c2 = hist(sys.argv[2])
        print(f"total {n} -> {n2} ({n2 - n:+d})")
        for k in sorted(set(c) | set(c2), key=lambda k: -(c2[k] - c[k]) ** 2):
            if c2[k] != c[k]:
                print(f"  {k:10s} {c[k]:5d} -> {c2[k]:5d} ({c2[k] - c[k]:+d})")
    else:
        print(f"total {n}")
        for k, v in c.most_common(30):
            print(f"  {k:10s} {v}")


if __name__ == "__main__":
    main()
