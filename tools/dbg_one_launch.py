import sys
sys.path.insert(0, "tests"); sys.path.insert(0, ".")
import numpy as np, torch, oracle, synth
from test_gpu_p2p_fused import Bands, DEFAULT
W, H, G = 1920, 1080, 2
b = Bands(W, H, G)
img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 201)
ref, S, _ = oracle.sharpen(img, *DEFAULT)
for ep in range(1, 5):
    out, sums = b.run(img, ep, fused=False, one_launch=True)
    bad = np.argwhere(out != ref)
    # halo contents
    b0, b1 = b.bands
    lower_halo0 = b0.band.cpu().numpy()[-4:]   # band 0's input includes rows up to row1+4
    upper_halo1 = b1.band.cpu().numpy()[:4]
    print(ep, sums == [S]*G, len(bad), bad[:3].tolist(),
          np.array_equal(lower_halo0, img[540:544]), np.array_equal(upper_halo1, img[536:540]), b.cap1)
b.close()
