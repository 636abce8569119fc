"""Phase timeline of single-image step launches (needs a library built with
-DSHARP_DIAG_TIMELINE, copied over libsharp.so).  Prints, per size, the median
over repetitions of each phase's globaltimer offset (us) from the first CTA's
start, plus the host-side event time of the call."""
import ctypes
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener, lib  # noqa: E402

L = lib()
L.sharp_debug_timeline.argtypes = [ctypes.c_void_p, ctypes.c_int]
names = ["start", "p1_first", "p1_last_end", "lut_first", "lut_last_end", "p2_first", "p2_last_end", "exit_last"]
buf = (ctypes.c_ulonglong * 8)()
for W, H in [(512, 512), (1920, 1080), (3840, 2160), (7680, 4320)]:
    s = Sharpener()
    s.set_path(1)  # the step kernel (the timeline probes live there)
    d = torch.from_numpy(synth.image(W, H, "natural", seed=1)).cuda()
    o = torch.empty_like(d)
    rows = []
    for it in range(30):
        L.sharp_debug_timeline(buf, 1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        s.enqueue_batch(d[None], o[None])
        e1.record()
        torch.cuda.synchronize()
        L.sharp_debug_timeline(buf, 0)
        v = [int(x) for x in buf]
        if it >= 5:
            rows.append([(x - v[0]) / 1e3 for x in v] + [e0.elapsed_time(e1) * 1e3])
    med = np.median(np.array(rows), axis=0)
    print(f"{W}x{H}: " + "  ".join(f"{n}={m:.1f}" for n, m in zip(names + ["event_us"], med)))
    s.close()
