#!/usr/bin/env python
"""Attribute dynamic SASS instruction counts (from an ncu report) to source
lines, using `nvdisasm -gi` line info of the same cubin.

usage: tools/sass_attrib.py REPORT.ncu-rep KERNEL.sass PIXELS [FUNC_SUBSTR]
  KERNEL.sass: nvdisasm -gi -c output of the cubin holding the kernel.
Prints thread-instructions per pixel grouped by (outermost kernel line,
innermost line)."""
import collections
import csv
import io
import re
import subprocess
import sys

rep, sassf, px = sys.argv[1], sys.argv[2], float(sys.argv[3])
fsub = sys.argv[4] if len(sys.argv) > 4 else "step_kernel"
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ia, isrc, iex = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
recs = [(int(r[ia], 16), r[isrc].strip(), int(r[iex] or 0)) for r in rows[2:] if len(r) > iex]
base = recs[0][0]
ex = {a - base: (s, e) for a, s, e in recs}

inner = outer = None
attr = {}
infunc = False
for line in open(sassf):
    if line.startswith(".text.") or "//----" in line:
        infunc = fsub in line
    if not infunc:
        continue
    m = re.match(r'\s*//## File "([^"]+)", line (\d+)(?: inlined at "([^"]+)", line (\d+))?', line)
    if m:
        f = m.group(1).split("/")[-1]
        if m.group(3) is None:
            outer = f"{f}:{m.group(2)}"
            if inner is None or not pending:
                inner = outer
            pending = False
        else:
            inner = f"{f}:{m.group(2)}"
            pending = True
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m:
        attr[int(m.group(1), 16)] = (outer, inner)
        pending = False
by = collections.Counter()
by_outer = collections.Counter()
for a, (o, i) in attr.items():
    if a in ex:
        by[(o, i)] += ex[a][1]
        by_outer[o] += ex[a][1]
tot = sum(by.values())
print(f"total {32 * tot / px:.2f} thread-instr/px")
print("-- by kernel line")
for k, v in by_outer.most_common(30):
    print(f"  {k:24s} {32 * v / px:6.2f}/px")
print("-- by (kernel line, innermost line)")
for k, v in by.most_common(50):
    print(f"  {k[0]:22s} {k[1]:28s} {32 * v / px:6.2f}/px")
