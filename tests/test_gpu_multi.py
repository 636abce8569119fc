"""Multi-device contexts (include/sharp.h sharp_config.num_devices / device_ids
/ shard): frames split over the devices, one image
as row bands (the L174 mean from the devices' partial sums), and
device-resident bands (sharp_run_bands), bit-exact vs the CPU oracle.  On a
one-GPU box every "device" is device 0 (device_ids = [0, 0, ...]): the same
sharding, halo and partial-sum code runs with separate per-entry contexts."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_EUNSUPPORTED, SHARP_SHARD_FRAMES, SHARP_SHARD_NONE,
                                            SHARP_SHARD_ROWS, SharpError, Sharpener, sharp_band_rows)

pytestmark = pytest.mark.gpu
PRM = (1.5, 0.5, 0.5, 2.0)


def ids(G):
    n = torch.cuda.device_count()
    return [g % n for g in range(G)]


@pytest.mark.parametrize("G", [2, 3])
@pytest.mark.parametrize("pinned", [False, True])
def test_frames_split_over_devices(G, pinned):
    n, W, H = 7, 640, 360
    imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 11)
    src = torch.from_numpy(imgs)
    if pinned:
        src = src.pin_memory()
    out = torch.empty_like(src)
    if pinned:
        out = out.pin_memory()
    with Sharpener(device_ids=ids(G), shard=SHARP_SHARD_FRAMES) as sh:
        sh.run_batch(src, PRM, out)
        sums = sh.batch_sums(n)
        st = sh.stats()
    ref, S = oracle.sharpen_batch(imgs, *PRM)
    assert np.array_equal(out.numpy(), ref)
    assert list(sums) == list(S)
    assert st.frames == n and st.edge_sum == S[0]


@pytest.mark.parametrize("G", [2, 3, 4])
@pytest.mark.parametrize("WH", [(1920, 1080), (3840, 2160), (512, 520)])
def test_one_image_as_row_bands(G, WH):
    W, H = WH
    img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 3)
    with Sharpener(device_ids=ids(G), shard=SHARP_SHARD_ROWS) as sh:
        out = sh.run(img, PRM)
        st = sh.stats()
    ref, S, mean = oracle.sharpen(img, *PRM)
    assert st.edge_sum == S and st.edge_mean == mean
    bad = np.argwhere(out != ref)
    assert bad.size == 0, f"{len(bad)} mismatches, first {bad[:3].tolist()}"


@pytest.mark.parametrize("G", [2, 3, 5])
def test_device_resident_bands(G):
    W, H = 1920, 1080
    img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 4)
    dev = ids(G)
    bands, outs = [], []
    for g in range(G):
        r0, r1 = sharp_band_rows(H, G, g)
        bands.append(torch.from_numpy(img[r0:r1].copy()).to(f"cuda:{dev[g]}"))
        outs.append(torch.empty_like(bands[-1]))
    with Sharpener(device_ids=dev) as sh:
        sh.run_bands(bands, W, H, PRM, outs)
        st = sh.stats()
    ref, S, _ = oracle.sharpen(img, *PRM)
    got = np.concatenate([o.cpu().numpy() for o in outs])
    assert st.edge_sum == S
    assert np.array_equal(got, ref)


def test_single_device_context_takes_one_band():
    W, H = 960, 540
    img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 9)
    d = torch.from_numpy(img).cuda()
    o = torch.empty_like(d)
    with Sharpener() as sh:
        sh.run_bands([d], W, H, PRM, [o])
    ref, _, _ = oracle.sharpen(img, *PRM)
    assert np.array_equal(o.cpu().numpy(), ref)


def test_shard_none_and_auto():
    W, H = 640, 360
    imgs = synth.frames(3, W, H, "natural", seed=synth.BASE_SEED + 12)
    ref, _ = oracle.sharpen_batch(imgs, *PRM)
    with Sharpener(device_ids=ids(2), shard=SHARP_SHARD_NONE) as sh:
        assert np.array_equal(sh.run_batch(imgs, PRM), ref)
    with Sharpener(device_ids=ids(2)) as sh:  # AUTO: frames for a batch, rows for one image
        assert np.array_equal(sh.run_batch(imgs, PRM), ref)
        assert np.array_equal(sh.run(imgs[1], PRM), ref[1])


def test_multi_device_context_rejects_device_buffers_and_async_calls():
    W, H = 640, 360
    d = torch.zeros((2, H, W), dtype=torch.uint8, device="cuda")
    o = torch.empty_like(d)
    with Sharpener(device_ids=ids(2)) as sh:
        with pytest.raises(SharpError) as e:
            sh.run_batch(d, PRM, o)
        assert e.value.code == SHARP_EUNSUPPORTED
        with pytest.raises(SharpError) as e:
            sh.enqueue_batch(d, o, PRM)
        assert e.value.code == SHARP_EUNSUPPORTED
