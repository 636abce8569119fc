"""Small invocations of every path for compute-sanitizer (tools/gpu_sanitize.sh):
the step kernel (batch + single image + a row band + the fused one-launch
band modes), the TMEM-resident kernel, the two-pass, scalar fused and staged
paths, the general-layout path and the reading switches, a multi-device
context; checked against the oracle so a sanitizer-perturbed run still has
to be right."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import (SHARP_PATH_FUSED, SHARP_PATH_FUSED_EXP, SHARP_PATH_RES,  # noqa: E402
                                            SHARP_PATH_STAGED, SHARP_PATH_STEP, SHARP_PATH_TWO_PASS, Sharpener,
                                            bands)
from paper_conf_icpp_fanjzac15_b200.bands import P2PBand, band_rows  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import sharp_p2p_window_create, sharp_p2p_window_destroy  # noqa: E402

imgs = synth.frames(3, 480, 64, "natural", seed=synth.BASE_SEED + 3)
ref, _ = oracle.sharpen_batch(imgs)
d = torch.from_numpy(imgs).cuda()
for path in (SHARP_PATH_STEP, SHARP_PATH_RES, SHARP_PATH_TWO_PASS, SHARP_PATH_FUSED, SHARP_PATH_FUSED_EXP,
             SHARP_PATH_STAGED):
    s = Sharpener()
    s.set_path(path)
    o = s.run_batch(d)
    torch.cuda.synchronize()
    assert np.array_equal(o.cpu().numpy(), ref), path
    s.close()
# a batch big enough for the step kernel's lagged schedule with multi-stage
# pass-1 and pass-2 tasks (>= one 2-sub-tile / 4-sub-tile task per CTA)
big = synth.frames(80, 480, 256, "natural", seed=synth.BASE_SEED + 4)
s = Sharpener()
s.set_path(SHARP_PATH_STEP)
o = s.run_batch(torch.from_numpy(big).cuda())
torch.cuda.synchronize()
assert np.array_equal(o.cpu().numpy(), oracle.sharpen_batch(big)[0]), "step lagged batch"
s.close()
s = Sharpener()
o = s.run(d[0])
torch.cuda.synchronize()
assert np.array_equal(o.cpu().numpy(), ref[0])
roi = d[:, 1:62, 3:470]
o = s.run_ex(roi, flags=oracle.READ_TRUNCATE | oracle.READ_INTERIOR_MEAN)
torch.cuda.synchronize()
for f in range(3):
    r, _, _ = oracle.sharpen_ex(imgs[f, 1:62, 3:470], flags=oracle.READ_TRUNCATE | oracle.READ_INTERIOR_MEAN)
    assert np.array_equal(o[f].cpu().numpy(), r)
out, _ = bands.sharpen_band(s, d[0], 480, 64, 0, 64)
torch.cuda.synchronize()
assert np.array_equal(out.cpu().numpy(), ref[0])
s.close()
# multi-device context (both entries on device 0): frames and row bands
m = Sharpener(device_ids=[0, 0])
assert np.array_equal(m.run_batch(imgs), ref)
assert np.array_equal(m.run(imgs[1]), ref[1])
m.close()
# fused band modes: 2 bands of one image on one device, peer-memory exchange in the step kernel
# (not under initcheck: it serialises kernels, and these two wait on each other)
if os.environ.get("SANITIZE_TOOL") == "initcheck":
    print("sanitize workload ok (fused band modes skipped under initcheck)")
    sys.exit(0)
W, H, G = 480, 64, 2
sms = torch.cuda.get_device_properties(0).multi_processor_count
shs = [Sharpener() for _ in range(G)]
sts = [torch.cuda.Stream() for _ in range(G)]
for sh_, st_ in zip(shs, sts):
    sh_.set_stream(st_)
wins = [sharp_p2p_window_create(W, band_rows(H, G, g)[1] - band_rows(H, G, g)[0]) for g in range(G)]
pbs = [P2PBand(shs[g], W, H, rank=g, world=G, window=wins[g], windows=wins) for g in range(G)]
for pb in pbs:  # every context's scratch first: an allocation may wait for the other band's spinning kernel
    tmp = torch.zeros(1, dtype=torch.int64, device="cuda")
    pb.sh.band_edge_sum(pb.band, W, H, pb.row0, pb.row1, tmp)
torch.cuda.synchronize()
for epoch, mode in enumerate(["fused", "one"], start=1):
    outs = []
    for pb, st_ in zip(pbs, sts):
        with torch.cuda.stream(st_):
            pb.own.copy_(d[0, pb.row0:pb.row1])
    torch.cuda.synchronize()
    for pb, st_ in zip(pbs, sts):
        with torch.cuda.stream(st_):
            o = torch.empty((pb.rows_own, W), dtype=torch.uint8, device="cuda")
            if mode == "fused":
                pb.step_fused(epoch, o, grid_cap=sms)
            else:
                pb.step_one_launch(epoch, o, grid_cap=sms)
            outs.append(o)
    torch.cuda.synchronize()
    assert np.array_equal(torch.cat(outs).cpu().numpy(), ref[0]), mode
for pb in pbs:
    pb.close()
for sh_ in shs:
    sh_.close()
print("sanitize workload ok")
