#!/usr/bin/env python
"""Per-SASS-instruction execution counts from an ncu report (source page):
opcode histogram and the hottest straight-line blocks.

usage: tools/sass_hot.py REPORT.ncu-rep [PIXELS] [--dump N]
"""
import collections
import csv
import io
import subprocess
import sys


def load(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    ia, isrc, iex, ist = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed"), \
        hdr.index("Warp Stall Sampling (All Samples)")
    recs = []
    for r in rows[2:]:
        if len(r) <= iex:
            continue
        recs.append((int(r[ia], 16), r[isrc].strip(), int(r[iex] or 0), int(r[ist] or 0)))
    return recs


def main():
    rep = sys.argv[1]
    px = float(sys.argv[2]) if len(sys.argv) > 2 and not sys.argv[2].startswith("-") else None
    recs = load(rep)
    tot = sum(e for _, _, e, _ in recs)
    samp = sum(s for _, _, _, s in recs) or 1
    print(f"instructions executed (warp): {tot:,}" + (f"  per px: {tot / px:.3f}" if px else ""))
    ops = collections.Counter()
    for _, s, e, _ in recs:
        op = s.split()[0] if s else "?"
        if op.startswith("@"):
            op = s.split()[1]
        ops[op.split(".")[0]] += e
    for op, e in ops.most_common(40):
        print(f"  {op:12s} {e / tot:6.1%}" + (f"  {e / px:.3f}/px" if px else ""))
    if "--dump" in sys.argv:
        n = int(sys.argv[sys.argv.index("--dump") + 1])
        base = recs[0][0]
        for a, s, e, st in recs:
            if e >= n:
                print(f"{a - base:6x} {e:12,d} {st:6d} {s}")


if __name__ == "__main__":
    main()
