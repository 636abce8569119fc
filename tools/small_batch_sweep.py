"""Per-call time of device run_batch for short batches of 1080p frames under
the lag policies (SHARP_EXP_LAG_POLICY, kernels_tma.cu): one JSON line per
(policy, n).  SWEEP_N / SWEEP_POL: comma-separated batch sizes / policies."""
import json
import os
import subprocess
import sys

if len(sys.argv) > 1 and sys.argv[1] == "worker":
    import time

    import numpy as np
    import torch
    sys.path.insert(0, ".")
    import synth
    from paper_conf_icpp_fanjzac15_b200 import Sharpener
    s = Sharpener()
    st = torch.cuda.Stream()
    s.set_stream(st)
    for n in [int(x) for x in os.environ.get('SWEEP_N', '1,2,4,6,8,12').split(',')]:
        d = torch.from_numpy(synth.frames(n, 1920, 1080, "natural", seed=5)).cuda()
        o = torch.empty_like(d)
        for _ in range(5):
            s.enqueue_batch(d, o)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(50):
            s.enqueue_batch(d, o)
        e1.record(st)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 50
        print(json.dumps({"policy": os.environ.get("SHARP_EXP_LAG_POLICY"), "n": n, "us": 1e3 * ms,
                          "gpx_s": n * 1920 * 1080 / ms / 1e6}), flush=True)
else:
    for pol in os.environ.get("SWEEP_POL", "1,2,3").split(","):
        subprocess.run([sys.executable, __file__, "worker"], env=dict(os.environ, SHARP_EXP_LAG_POLICY=pol))
