"""Where the single-image e2e time goes (1080p, pinned host buffers):
(a) H2D + D2H copies only, (b) H2D + enqueue_batch + D2H on one stream,
(c) sharp_run on the pinned buffers (the public API).  Median wall us of 200."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402
from paper_conf_icpp_fanjzac15_b200.binding import _params  # noqa: E402

for W, H in [(1920, 1080), (3840, 2160)]:
    h_in = torch.from_numpy(synth.image(W, H, "natural", seed=1)).pin_memory()
    h_out = torch.empty_like(h_in).pin_memory()
    d_in = torch.empty((1, H, W), dtype=torch.uint8, device="cuda")
    d_out = torch.empty_like(d_in)
    st = torch.cuda.Stream()
    s = Sharpener()
    s.set_stream(st)
    prm = _params((1.0, 0.5, 0.5, 2.0))

    def a():
        with torch.cuda.stream(st):
            d_in.view(H, W).copy_(h_in, non_blocking=True)
            h_out.copy_(d_in.view(H, W), non_blocking=True)
        st.synchronize()

    def b():
        with torch.cuda.stream(st):
            d_in.view(H, W).copy_(h_in, non_blocking=True)
            s.enqueue_batch(d_in, d_out, prm)
            h_out.copy_(d_out.view(H, W), non_blocking=True)
        st.synchronize()

    s2 = Sharpener()

    def c():
        s2.run(h_in, prm, h_out)

    for name, fn in [("copies", a), ("copies+enqueue", b), ("sharp_run", c)]:
        for _ in range(20):
            fn()
        ts = []
        for _ in range(200):
            t0 = time.perf_counter()
            fn()
            ts.append(time.perf_counter() - t0)
        print(f"{W}x{H} {name}: {1e6 * np.median(ts):.1f} us")
    s.close()
    s2.close()
