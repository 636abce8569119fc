"""Host vs device time per single-image call (enqueue_batch loop): if the host
wall time per call is >= the device time per call, the single-image path is
host-bound."""
import sys
import time

import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

for W, H in [(512, 512), (1920, 1080)]:
    s = Sharpener()
    st = torch.cuda.Stream()
    s.set_stream(st)
    d = torch.from_numpy(synth.image(W, H, "natural", seed=1)).cuda()[None]
    o = torch.empty_like(d)
    for _ in range(50):
        s.enqueue_batch(d, o)
    torch.cuda.synchronize()
    n = 500
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    t0 = time.perf_counter()
    for _ in range(n):
        s.enqueue_batch(d, o)
    t1 = time.perf_counter()
    e1.record(st)
    torch.cuda.synchronize()
    print(f"{W}x{H}: host {1e6 * (t1 - t0) / n:.1f} us/call, device {1e3 * e0.elapsed_time(e1) / n:.1f} us/call")
    s.close()
