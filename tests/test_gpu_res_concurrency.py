"""The TMEM-resident kernel's static schedule needs all of its CTAs resident
at once; it is launched cooperatively, so two of them on concurrent streams
(or beside a persistent step kernel) complete instead of each holding part of
the SMs.  Also: SHARP_PATH_AUTO picks it for mid-size launches and the step
kernel for big ones, both bit-exact."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import SHARP_PATH_RES, SHARP_PATH_STEP, Sharpener

pytestmark = pytest.mark.gpu
PRM = (1.0, 0.5, 0.5, 2.0)


@pytest.mark.parametrize("other", [SHARP_PATH_RES, SHARP_PATH_STEP])
def test_two_streams_concurrently(other):
    n, W, H = 6, 1920, 1080
    imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 31)
    ref, _ = oracle.sharpen_batch(imgs, *PRM)
    d = torch.from_numpy(imgs).cuda()
    outs, shs, sts = [], [], []
    for path in (SHARP_PATH_RES, other):
        st = torch.cuda.Stream()
        sh = Sharpener()
        sh.set_stream(st)
        sh.set_path(path)
        shs.append(sh)
        sts.append(st)
        outs.append(torch.empty_like(d))
    torch.cuda.synchronize()
    for _ in range(5):  # interleaved launches on the two streams
        for sh, o in zip(shs, outs):
            sh.enqueue_batch(d, o, PRM)
    torch.cuda.synchronize()
    for o in outs:
        assert np.array_equal(o.cpu().numpy(), ref)
    for sh in shs:
        sh.close()


@pytest.mark.parametrize("n,W,H", [(1, 1920, 1080), (3, 3840, 2160), (40, 1280, 720), (1, 512, 512), (64, 1920, 1080)])
def test_auto_choice_is_exact(n, W, H):
    imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 32)
    ref, sums = oracle.sharpen_batch(imgs, *PRM)
    d = torch.from_numpy(imgs).cuda()
    with Sharpener() as sh:
        o = torch.empty_like(d)
        sh.run_batch(d, PRM, o)
        assert np.array_equal(o.cpu().numpy(), ref)
        assert sh.batch_sums(n) == [int(x) for x in sums]
