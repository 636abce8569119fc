"""Run one sharpen on a synthetic WxH image through the C ABI and compare with the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

W, H = int(sys.argv[1]), int(sys.argv[2])
n = int(sys.argv[3]) if len(sys.argv) > 3 else 1
imgs = synth.frames(n, W, H, "natural", seed=W * 1000 + H)
with Sharpener() as s:
    d = torch.from_numpy(imgs).cuda()
    o = torch.empty_like(d)
    s.run_batch(d, (1.0, 0.5, 0.5, 2.0), o)
    torch.cuda.synchronize()
    sums = s.batch_sums(n)
ref, rs = oracle.sharpen_batch(imgs)
out = o.cpu().numpy()
bad = np.argwhere(out != ref)
print("sums ok", list(map(int, rs)) == sums, "mismatches", len(bad), bad[:10].tolist())
