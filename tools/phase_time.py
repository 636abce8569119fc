#!/usr/bin/env python
"""Single-image phase split (diagnostic): tools/phase_time.py [W H]
Times, on one stream, back-to-back: the whole image (sharp_enqueue_batch,
AUTO), pass 1 alone (sharp_band_edge_sum over all rows), pass 2 alone
(sharp_band_sharpen with the total precomputed), and an empty kernel launch."""
import sys
import torch
sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener, binding as B  # noqa: E402

W = int(sys.argv[1]) if len(sys.argv) > 1 else 7680
H = int(sys.argv[2]) if len(sys.argv) > 2 else 4320
img = torch.from_numpy(synth.frames(1, W, H, "natural", seed=synth.BASE_SEED + 5)).cuda()  # [1, H, W]
out = torch.empty_like(img)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
sh = Sharpener()
sh.set_stream(st)
ctx = sh.ctx
part = torch.zeros(1, dtype=torch.int64, device="cuda")
prm = (1.0, 0.5, 0.5, 2.0)


def timeit(f, reps=200):
    for _ in range(5):
        f()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(reps):
        f()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


def graph_time(f, reps=100):
    f()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        for _ in range(reps):
            f()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(5):
        g.replay()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / (5 * reps) * 1e3


for path in (1, 0):
    sh.set_path(path)
    t = timeit(lambda: sh.enqueue_batch(img, out, prm))
    tg = graph_time(lambda: sh.enqueue_batch(img, out, prm))
    print(f"whole image path {path}: {t:.1f} us (graph {tg:.1f} us)")
sh.set_path(1)
t1 = timeit(lambda: B.sharp_band_edge_sum(ctx, img[0], W, H, 0, H, part))
torch.cuda.synchronize()
t2 = timeit(lambda: B.sharp_band_sharpen(ctx, img[0], W, H, 0, H, part, prm, out[0]))
z = torch.zeros(1, device="cuda")
t0 = timeit(lambda: z.add_(1))
print(f"pass 1 alone: {t1:.1f} us   pass 2 alone: {t2:.1f} us   sum {t1 + t2:.1f}   empty launch {t0:.1f} us")
