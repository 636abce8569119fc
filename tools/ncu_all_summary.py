"""Per-kernel summary of an ncu launch list with duration + DRAM bytes
(tools/gpu_ncu_all.sh): launches, mean duration, DRAM GB/s and % of the HBM
peak (MEASURED_PEAKS.json), as markdown.

usage: tools/ncu_all_summary.py ALL_KERNELS.csv > profiles/<round>/ncu_all_kernels.md"""
import collections
import csv
import json
import os
import re
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ik, im, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
ii = hdr.index("ID")
per = collections.defaultdict(dict)
names = {}
for r in rows[1:]:
    v = float(r[iv].replace(",", ""))
    unit = r[iu]
    if r[im].startswith("dram__bytes"):
        v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
    elif r[im] == "gpu__time_duration.sum":
        v *= {"ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3}.get(unit, 1e-9)
    per[r[ii]][r[im]] = v
    names[r[ii]] = re.sub(r"\(.*", "", r[ik].replace("<unnamed>::", "").replace("(anonymous namespace)::", ""))
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
try:
    peak = float(json.load(open(os.path.join(root, "MEASURED_PEAKS.json")))["hbm_gbs"])
    src = "MEASURED_PEAKS.json"
except (OSError, KeyError, ValueError):
    peak, src = 8000.0, "fallback"
print("# ncu: every kernel of libsharp.so (tools/all_kernels_workload.py, 4K frames)\n")
print(f"Cold-cache, serialised launches (ncu replays each kernel, so the input written just before a "
      f"launch can still sit in L2: DRAM bytes below the algorithmic ones mean L2 hits); HBM peak "
      f"{peak:.0f} GB/s ({src}).  The step kernel's batch-scale numbers are in ncu_summary.md.\n")
print("| # | kernel | duration (us) | DRAM read + write (MB) | DRAM GB/s | % of HBM peak |")
print("|---|---|---|---|---|---|")
for i in sorted(per, key=int):
    d, n = per[i], names[i]
    if n.startswith("void at::"):
        continue  # torch fill kernels of the test harness
    t = d.get("gpu__time_duration.sum", 0.0)
    b = d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
    gbs = b / t / 1e9 if t else 0.0
    print(f"| {i} | `{n}` | {1e6 * t:.1f} | {b / 1e6:.2f} | {gbs:.0f} | {100 * gbs / peak:.1f}% |")
