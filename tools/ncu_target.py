"""Small fixed workload for ncu captures: 24 x 1080p frames (two chunks of 12),
enqueued `reps` times on one stream."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--frames", type=int, default=24)
ap.add_argument("--width", type=int, default=1920)
ap.add_argument("--height", type=int, default=1080)
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
imgs = synth.frames(a.frames, a.width, a.height, "natural", seed=synth.BASE_SEED + 5)
d = torch.from_numpy(imgs).cuda()
o = torch.empty_like(d)
with Sharpener() as s:
    for _ in range(a.reps):
        s.enqueue_batch(d, o, (1.0, 0.5, 0.5, 2.0))
    torch.cuda.synchronize()
print("done", s is not None)
