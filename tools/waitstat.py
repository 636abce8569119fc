"""Timing experiment: consumer full-barrier wait cycles by (previous, awaited)
task type (needs a libsharp.so built with -DSHARP_EXP_WAITSTAT)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener, lib  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
imgs = synth.frames(n, 1920, 1080, "natural", seed=synth.BASE_SEED + 5)
d = torch.from_numpy(imgs).cuda()
o = torch.empty_like(d)
arr = (ctypes.c_ulonglong * 80)()
f = lib().sharp_debug_waitstat
with Sharpener() as s:
    s.enqueue_batch(d, o)
    torch.cuda.synchronize()
    f(arr, 1)
    s.enqueue_batch(d, o)
    torch.cuda.synchronize()
    f(arr, 1)
names = ["empty", "P1", "LUT", "P2", "end"]
total = arr[50]
print(f"consumer-warp cycles (sum over warps): {total:.3e}")
rows = []
for p in range(5):
    for c in range(5):
        cyc, cnt = arr[(p * 5 + c) * 2], arr[(p * 5 + c) * 2 + 1]
        if cnt:
            rows.append((cyc, f"prev {names[p]:5s} -> {names[c]:5s}: waits {cnt:9d}  cycles {cyc:.3e} ({cyc / total:6.2%})  avg {cyc / cnt:8.0f}"))
for _, r in sorted(rows, reverse=True):
    print(r)
for c in range(5):
    cnt = arr[(26 + c) * 2 + 1]
    if cnt:
        print(f"{names[c]:5s}: when warp 0 had to wait, issue->completion latency avg {arr[(26 + c) * 2] / cnt:8.0f} cycles ({cnt} waits)")
