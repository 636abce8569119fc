"""Randomised parameter stress of bit-exact parity (R19: CUDA's f64
pow / exp vs glibc, rounded to f32): N seeded random (A, gamma, G, K) sets x
rotating natural / noise frames, every output compared with the oracle.
Prints one JSON line {cases, pixels, mismatched_pixels, mismatched_cases}."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
rng = np.random.default_rng(2015)
s = Sharpener()
imgs = [synth.image(128, 64, ["natural", "noise"][i % 2], seed=synth.BASE_SEED + 7000 + i) for i in range(16)]
d = [torch.from_numpy(im).cuda() for im in imgs]
o = torch.empty_like(d[0])
bad_px = bad_cases = px = 0
first = None
for case in range(N):
    prm = tuple(float(np.float32(v)) for v in (rng.uniform(0, 16), rng.uniform(0, 4), rng.uniform(0, 1),
                                                np.exp(rng.uniform(np.log(1e-3), np.log(1e6)))))
    k = case % len(imgs)
    s.run(d[k], prm, o)
    ref, _, _ = oracle.sharpen(imgs[k], *prm)
    got = o.cpu().numpy()
    nb = int((got != ref).sum())
    px += got.size
    if nb:
        bad_px += nb
        bad_cases += 1
        first = first or {"case": case, "params": prm, "frame": k}
print(json.dumps({"cases": N, "pixels": px, "mismatched_pixels": bad_px, "mismatched_cases": bad_cases,
                  "first": first}))
