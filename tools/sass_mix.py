"""Aggregate an `ncu --page source --print-source sass --csv` dump by opcode
(dynamic warp-instruction counts) and by code region."""
import csv
import re
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
iexe = hdr.index("Instructions Executed")
src = hdr.index("Source")
stall = hdr.index("Warp Stall Sampling (All Samples)")
px = float(sys.argv[2]) if len(sys.argv) > 2 else None
ops, total, stalls = Counter(), 0, Counter()
for r in rows[2:]:
    if len(r) <= iexe or not r[iexe]:
        continue
    n = int(r[iexe])
    s = r[src].strip()
    m = re.match(r"(@!?U?P\w+\s+)?([A-Z0-9_]+)(\.[A-Z0-9_.]+)?", s)
    op = m.group(2) if m else s.split()[0]
    ops[op] += n
    stalls[op] += int(r[stall] or 0)
    total += n
print(f"total warp-instructions {total}" + (f"  -> {32 * total / px:.2f} thread-instr/px" if px else ""))
for op, n in ops.most_common(40):
    print(f"{op:12s} {n:10d} {100 * n / total:5.1f}%" + (f"  {32 * n / px:6.2f}/px" if px else "") + f"  stall-samples {stalls[op]}")
