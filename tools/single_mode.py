#!/usr/bin/env python
"""One W x H image, MODE = whole | p1 | p2, REPS back-to-back calls (for ncu
captures of a single-image launch): tools/single_mode.py MODE [W H REPS]"""
import sys
import torch
sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener, binding as B  # noqa: E402

mode = sys.argv[1]
W = int(sys.argv[2]) if len(sys.argv) > 2 else 7680
H = int(sys.argv[3]) if len(sys.argv) > 3 else 4320
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 5
img = torch.from_numpy(synth.frames(1, W, H, "natural", seed=synth.BASE_SEED + 5)).cuda()
out = torch.empty_like(img)
sh = Sharpener()
sh.set_path(1)
part = torch.zeros(1, dtype=torch.int64, device="cuda")
prm = (1.0, 0.5, 0.5, 2.0)
B.sharp_band_edge_sum(sh.ctx, img[0], W, H, 0, H, part)
for _ in range(reps):
    if mode == "whole":
        sh.enqueue_batch(img, out, prm)
    elif mode == "p1":
        B.sharp_band_edge_sum(sh.ctx, img[0], W, H, 0, H, part)
    else:
        B.sharp_band_sharpen(sh.ctx, img[0], W, H, 0, H, part, prm, out[0])
torch.cuda.synchronize()
