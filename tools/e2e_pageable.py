"""sharp_run_batch e2e with PAGEABLE host buffers (numpy), 256 x 1080p: median
wall ms of 3 calls -> Gpx/s."""
import json
import sys
import time

import numpy as np

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

N = 256
imgs = synth.frames(N, 1920, 1080, "natural", seed=1)
out = np.empty_like(imgs)
s = Sharpener()
s.run_batch(imgs, None, out)
ts = []
for _ in range(3):
    t0 = time.perf_counter()
    s.run_batch(imgs, None, out)
    ts.append(time.perf_counter() - t0)
ms = 1e3 * float(np.median(ts))
print(json.dumps({"frames": N, "ms": ms, "gpx_s": N * 1920 * 1080 / ms / 1e6}))
