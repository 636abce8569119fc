"""Small invocations of every path for compute-sanitizer (tools/gpu_sanitize.sh):
the step kernel (batch + single image + a row band), the two-pass and staged
paths, the general-layout path and the reading switches; checked against the
oracle so a sanitizer-perturbed run still has to be right."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import (SHARP_PATH_STAGED, SHARP_PATH_STEP, SHARP_PATH_TWO_PASS,  # noqa: E402
                                            Sharpener, bands)

imgs = synth.frames(3, 480, 64, "natural", seed=synth.BASE_SEED + 3)
ref, _ = oracle.sharpen_batch(imgs)
d = torch.from_numpy(imgs).cuda()
for path in (SHARP_PATH_STEP, SHARP_PATH_TWO_PASS, SHARP_PATH_STAGED):
    s = Sharpener()
    s.set_path(path)
    o = s.run_batch(d)
    torch.cuda.synchronize()
    assert np.array_equal(o.cpu().numpy(), ref), path
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
print("sanitize workload ok")
