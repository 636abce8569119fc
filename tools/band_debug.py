"""Debug helper: per-band mismatch maps of the row-band path vs the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener, sharp_band_halo  # noqa: E402

W, H = int(sys.argv[1]), int(sys.argv[2])
rows = [tuple(map(int, r.split(":"))) for r in sys.argv[3:]]
img = synth.image(W, H, "natural", seed=W + H + len(rows))
ref, S_ref, _ = oracle.sharpen(img)
d = torch.from_numpy(img).cuda()
tot = torch.tensor([S_ref], dtype=torch.int64, device="cuda")
with Sharpener() as sh:
    for r0, r1 in rows:
        in0, in1 = sharp_band_halo(H, r0, r1)
        band = d[in0:in1].clone()
        o = torch.empty((r1 - r0, W), dtype=torch.uint8, device="cuda")
        sh.band_sharpen(band, W, H, r0, r1, tot, o)
        torch.cuda.synchronize()
        bad = np.argwhere(o.cpu().numpy() != ref[r0:r1])
        rr = np.unique(bad[:, 0] + r0) if len(bad) else []
        cc = np.unique(bad[:, 1]) if len(bad) else []
        print(f"band {r0}:{r1} in {in0}:{in1} mismatches {len(bad)} rows {list(rr[:40])} ncols {len(cc)} cols {list(cc[:20])}")
