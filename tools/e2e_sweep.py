"""Sweep the host pipeline (streams x chunk_frames) of sharp_run_batch on
pinned host buffers, 1024 x 1080p (the bench e2e leg).  One JSON line per
setting: median wall ms of 3 calls."""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

N, W, H = 1024, 1920, 1080
h_in = torch.empty((N, H, W), dtype=torch.uint8).pin_memory()
synth.frames(N, W, H, "natural", seed=synth.BASE_SEED + 5, out=h_in.numpy())
h_out = torch.empty_like(h_in).pin_memory()
for streams in [int(x) for x in sys.argv[1].split(",")]:
    for chunk in [int(x) for x in sys.argv[2].split(",")]:
        sh = Sharpener(streams=streams, chunk_frames=chunk)
        sh.run_batch(h_in, None, h_out)
        ts = []
        for _ in range(3):
            t0 = time.perf_counter()
            sh.run_batch(h_in, None, h_out)
            ts.append(time.perf_counter() - t0)
        ms = 1e3 * float(np.median(ts))
        print(json.dumps({"streams": streams, "chunk_frames": chunk, "ms": ms, "gpx_s": N * W * H / ms / 1e6}),
              flush=True)
        sh.close()
