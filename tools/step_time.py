#!/usr/bin/env python
"""Batch time of a given kernel path (A/B helper): tools/step_time.py PATH [FRAMES W H]
PATH: 1 = step kernel, 4 = resident kernel, 0 = auto."""
import sys
import torch
sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

path = int(sys.argv[1])
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
W = int(sys.argv[3]) if len(sys.argv) > 3 else 1920
H = int(sys.argv[4]) if len(sys.argv) > 4 else 1080
imgs = torch.from_numpy(synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 5)).cuda()
out = torch.empty_like(imgs)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
sh = Sharpener()
sh.set_stream(st)
sh.set_path(path)
prm = (1.0, 0.5, 0.5, 2.0)
reps = max(5, 2000 // n)
for _ in range(3):
    sh.enqueue_batch(imgs, out, prm)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record(st)
for _ in range(reps):
    sh.enqueue_batch(imgs, out, prm)
e1.record(st)
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
print(f"path {path} {n} x {W}x{H}: {ms:.4f} ms per call, {n * W * H / ms / 1e6:.1f} Gpx/s")
