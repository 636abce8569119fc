"""One small invocation of every kernel of libsharp.so, for an ncu launch
list (tools/gpu_ncu_all.sh): the step kernel, the two-pass kernels, the
staged K1..K7, the layout gather / scatter, the row-band kernels and the
peer-memory exchange kernels (1 band), on 4K frames."""
import sys

import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import (SHARP_PATH_STAGED, SHARP_PATH_STEP,  # noqa: E402
                                            SHARP_PATH_TWO_PASS, Sharpener, bands)

W, H, N = 3840, 2160, 4
imgs = torch.from_numpy(synth.frames(N, W, H, "natural", seed=synth.BASE_SEED + 2)).cuda()
out = torch.empty_like(imgs)
for path in (SHARP_PATH_STEP, SHARP_PATH_TWO_PASS, SHARP_PATH_STAGED):
    s = Sharpener()
    s.set_path(path)
    s.run_batch(imgs, None, out)
    s.close()
s = Sharpener()
roi = imgs[:, 1:H - 3, 5:W - 2]                      # pitched ROI, odd width: gather / run / scatter
s.run_ex(roi, out=torch.empty_like(roi))
torch.cuda.synchronize()
# the whole image as one row band: band calls (NCCL-free at one rank) ...
band_out, _ = bands.sharpen_band(s, imgs[0], W, H, 0, H)
# ... and the peer-memory exchange kernels (one band, single process)
pb = bands.P2PBand(s, W, H, rank=0, world=1)
pb.own.copy_(imgs[0])
pb.step(1, torch.empty((H, W), dtype=torch.uint8, device="cuda"))
torch.cuda.synchronize()
pb.close()
s.close()
torch.cuda.synchronize()
print("ok")
