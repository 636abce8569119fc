import sys, torch
sys.path.insert(0, ".")
import synth
from paper_conf_icpp_fanjzac15_b200 import Sharpener
s = Sharpener()
rgb = torch.from_numpy(synth.frames(24, 1920, 1080, "natural", seed=3).reshape(8, 3, 1080, 1920).transpose(0, 2, 3, 1).copy()).cuda()
o = torch.empty_like(rgb)
for _ in range(3):
    s.run_ex(rgb, out=o, channels_last=True)
torch.cuda.synchronize()
