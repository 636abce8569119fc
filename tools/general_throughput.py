"""Throughput of sharp_run_ex layouts on device buffers (median of 10 calls,
host wall clock around the synchronous call): dense batch (reference), an
aligned ROI (zero-copy), interleaved RGB (gather / scatter), a size that is
not a multiple of 4, and W % 16 == 8.  One JSON line per case."""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

s = Sharpener()
N = 32


def timeit(fn, px):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(10):
        t0 = time.perf_counter()
        fn()
        ts.append(time.perf_counter() - t0)
    ms = 1e3 * float(np.median(ts))
    return {"ms": ms, "gpx_s": px / ms / 1e6}


frames = torch.from_numpy(synth.frames(N, 1920, 1080, "natural", seed=synth.BASE_SEED + 1)).cuda()
out = torch.empty_like(frames)
cases = {}
cases["dense 32 x 1920x1080 (run_batch)"] = timeit(lambda: s.run_batch(frames, None, out), N * 1920 * 1080)
big = torch.from_numpy(synth.frames(N, 2048, 1100, "natural", seed=synth.BASE_SEED + 2)).cuda()
roi = big[:, 8:1088, 64:1984]
oroi = torch.empty_like(big)[:, 8:1088, 64:1984]
cases["aligned ROI 32 x 1920x1080 of 2048x1100 (zero-copy)"] = timeit(lambda: s.run_ex(roi, out=oroi), N * 1920 * 1080)
rgb = torch.from_numpy(synth.frames(3 * N // 4, 1920, 1080, "natural", seed=3).reshape(N // 4, 3, 1080, 1920)
                       .transpose(0, 2, 3, 1).copy()).cuda()
orgb = torch.empty_like(rgb)
cases["interleaved RGB 8 x 1920x1080x3 (gather/scatter)"] = timeit(
    lambda: s.run_ex(rgb, out=orgb, channels_last=True), 3 * (N // 4) * 1920 * 1080)
odd = frames[:, :1079, :1919]
oodd = torch.empty_like(frames)[:, :1079, :1919]
cases["odd size 32 x 1919x1079 (replicate-extend)"] = timeit(lambda: s.run_ex(odd, out=oodd), N * 1919 * 1079)
w8 = torch.from_numpy(synth.frames(N, 1928, 1080, "natural", seed=4)).cuda()
ow8 = torch.empty_like(w8)
cases["dense 32 x 1928x1080 (W % 16 == 8)"] = timeit(lambda: s.run_batch(w8, None, ow8), N * 1928 * 1080)
for k, v in cases.items():
    print(json.dumps({"case": k, **v}))
s.close()
