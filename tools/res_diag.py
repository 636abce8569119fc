#!/usr/bin/env python
"""Wait-cycle counters of the resident kernel (needs a libsharp.so built with
-DSHARP_DIAG_RES copied over the package's; diagnostics only).

usage: tools/res_diag.py [FRAMES] [W] [H]"""
import ctypes
import sys
import time

import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener, binding  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
W = int(sys.argv[2]) if len(sys.argv) > 2 else 1920
H = int(sys.argv[3]) if len(sys.argv) > 3 else 1080
lib = binding.lib()
diag = hasattr(lib, "sharp_debug_res")
buf = (ctypes.c_ulonglong * 16)()
imgs = torch.from_numpy(synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 5)).cuda()
out = torch.empty_like(imgs)
sh = Sharpener()
sh.set_path(4)  # SHARP_PATH_RES
for _ in range(2):
    sh.enqueue_batch(imgs, out, (1.0, 0.5, 0.5, 2.0))
torch.cuda.synchronize()
if diag:
    lib.sharp_debug_res(buf, 1)
t0 = time.perf_counter()
reps = 3
for _ in range(reps):
    sh.enqueue_batch(imgs, out, (1.0, 0.5, 0.5, 2.0))
torch.cuda.synchronize()
dt = (time.perf_counter() - t0) / reps
if not diag:
    print(f"{n} x {W}x{H}: {dt * 1e3:.3f} ms per batch ({n * W * H / dt / 1e9:.1f} Gpx/s)")
    sys.exit(0)
lib.sharp_debug_res(buf, 1)
v = [x / reps for x in buf]
mhz = 1965.0
print(f"res grid {lib.sharp_debug_res_grid()}; {n} x {W}x{H}: {dt * 1e3:.3f} ms per batch ({n * W * H / dt / 1e9:.1f} Gpx/s)")
print(f"P1 stage waits: {v[1]:.0f} x {v[0] / max(v[1], 1) / mhz:.3f} us (per consumer warp-0 lane... per warp)")
print(f"P2 stage waits: {v[3]:.0f} x {v[2] / max(v[3], 1) / mhz:.3f} us")
print(f"producer table waits total {v[4] / mhz / 1e3:.3f} ms-CTA, chunks built {v[5]:.0f}")
print(f"producer empty waits total {v[6] / mhz / 1e3:.3f} ms-CTA")
print(f"chunk build: {v[7] / max(v[5], 1) / mhz:.3f} us per chunk")
print(f"table done at first look: {v[8]:.0f}; saw pass 1 complete: {v[11]:.0f} x (wait pass1 {v[9] / max(v[11], 1) / mhz:.3f} us, then table {v[10] / max(v[11], 1) / mhz:.3f} us); waited w/o seeing: {v[12] / mhz / 1e3:.3f} ms")
print(f"P2 waits (warp 0, > 1000 cyc): {v[13]:.0f}; at wait end: {v[14] / max(v[13], 1) / mhz:.3f} us since tile TMA issue, {v[15] / max(v[13], 1) / mhz:.3f} us since table copy issue")
print(f"  producer lane 1 per table copy: acquire load {v[7] / 184320 / mhz:.3f} us, proxy fence {v[12] / 184320 / mhz:.3f} us (per P2 of a 1080p batch)")
occ = (ctypes.c_int * 8)()
lib.sharp_debug_res_occ(occ)
print("regs, static smem, max dyn smem, kResSmem, occ err, occ, occ(0 dyn), max threads:", list(occ))
