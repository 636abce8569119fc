#!/usr/bin/env python
"""Stall samples of an ncu report grouped by SASS address range and reason.

usage: tools/stall_regions.py REPORT.ncu-rep [TOP_N]
Prints the top instructions by samples (with their reasons) and the
per-reason totals."""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ia, isrc, isamp, iex = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)"), \
    hdr.index("Instructions Executed")
reasons = [(i, h) for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
recs = []
for r in rows[2:]:
    if len(r) <= iex:
        continue
    rs = {h: int(r[i] or 0) for i, h in reasons}
    recs.append((int(r[ia], 16), r[isrc].strip(), int(r[isamp] or 0), int(r[iex] or 0), rs))
base = recs[0][0]
tot = sum(x[2] for x in recs) or 1
print(f"total samples {tot}")
for a, s, n, e, rs in sorted(recs, key=lambda x: -x[2])[:top]:
    main = sorted(rs.items(), key=lambda kv: -kv[1])[:3]
    print(f"{a - base:6x} {n:7d} {100 * n / tot:5.2f}% ex={e:<12,d} {s[:60]:60s} " +
          " ".join(f"{k[6:]}={v}" for k, v in main if v))
