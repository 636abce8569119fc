"""Row-band sharding of one image on one GPU: every
band runs through the C ABI (sharp_band_edge_sum -> sum of the partials ->
sharp_band_sharpen) from a buffer holding only its rows plus the halo, and
the assembled bands must equal the whole-image oracle bit for bit (and the
summed partials its S).  The multi-rank plumbing (halo exchange, all-reduce)
is covered on CPU by tests/test_bands_cpu.py."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_EINVAL, SHARP_EUNSUPPORTED, SharpError, Sharpener,
                                            sharp_band_halo)
from paper_conf_icpp_fanjzac15_b200.bands import band_rows, halo_rows, sharpen_band

pytestmark = pytest.mark.gpu

DEFAULT = (1.0, 0.5, 0.5, 2.0)


@pytest.fixture(scope="module")
def sh():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    s = Sharpener()
    s.set_stream(torch.cuda.current_stream())  # the band calls are asynchronous: order them with torch's ops
    yield s
    s.close()


def run_bands(sh, img, rows, prm=DEFAULT):
    """rows: list of (row0, row1).  Returns (assembled output, S)."""
    H, W = img.shape
    d = torch.from_numpy(img).cuda()
    parts = torch.zeros(len(rows), dtype=torch.int64, device="cuda")
    bands = []
    for g, (r0, r1) in enumerate(rows):
        in0, in1 = sharp_band_halo(H, r0, r1)
        band = d[in0:in1].clone()  # only its rows + halo
        bands.append(band)
        sh.band_edge_sum(band, W, H, r0, r1, parts[g:g + 1])
    total = parts.sum().reshape(1)
    out = torch.full((H, W), 7, dtype=torch.uint8, device="cuda")
    for g, (r0, r1) in enumerate(rows):
        o = torch.empty((r1 - r0, W), dtype=torch.uint8, device="cuda")
        sh.band_sharpen(bands[g], W, H, r0, r1, total, o, prm)
        out[r0:r1] = o
    torch.cuda.synchronize()
    return out.cpu().numpy(), int(total.item()), parts.cpu().numpy()


def check(sh, img, rows, prm=DEFAULT):
    out, S, parts = run_bands(sh, img, rows, prm)
    ref, S_ref, _ = oracle.sharpen(img, *prm)
    assert S == S_ref
    pE = oracle.sobel(img)
    for g, (r0, r1) in enumerate(rows):  # each partial is its band's own rows
        assert parts[g] == int(pE[r0:r1].astype(np.int64).sum())
    bad = np.argwhere(out != ref)
    assert bad.size == 0, f"{len(bad)} mismatches, first {bad[:5].tolist()}"


@pytest.mark.parametrize("W,H,G", [(1920, 1080, 2), (1920, 1080, 3), (512, 512, 4), (256, 40, 10), (16, 16, 4),
                                   (3840, 2160, 4), (976, 212, 7)])
def test_bands_equal_whole_image(sh, W, H, G):
    img = synth.image(W, H, "natural", seed=W + H + G)
    check(sh, img, [band_rows(H, G, g) for g in range(G)])


@pytest.mark.parametrize("prm", [(1.0, 0.0, 0.5, 2.0), (2.5, 1.0, 0.25, 1.0), (16.0, 4.0, 1.0, 1e6)])
def test_bands_params(sh, prm):
    img = synth.image(1920, 1080, "noise", seed=3)
    check(sh, img, [band_rows(1080, 3, g) for g in range(3)], prm)


def test_uneven_band_boundaries(sh):
    """Bands starting at rows that are multiples of 4 but not of the tile
    heights (12 / 18), including 4-row bands at the image edges."""
    img = synth.image(480, 200, "natural", seed=11)
    check(sh, img, [(0, 4), (4, 8), (8, 40), (40, 44), (44, 196), (196, 200)])


def test_8k_bands_sampled(sh):
    """8K (BASELINE C4) at 8 bands; compared with the oracle on every pixel."""
    img = synth.image(7680, 4320, "natural", seed=8)
    check(sh, img, [band_rows(4320, 8, g) for g in range(8)])


def test_single_band_is_whole_image(sh):
    img = synth.image(1920, 1080, "natural", seed=5)
    out, S, _ = run_bands(sh, img, [(0, 1080)])
    ref, S_ref, _ = oracle.sharpen(img, *DEFAULT)
    assert S == S_ref and np.array_equal(out, ref)


def test_sharpen_band_world1(sh):
    """bands.sharpen_band without a process group: the whole image."""
    img = synth.image(960, 540, "natural", seed=9)
    d = torch.from_numpy(img).cuda()
    out, s = sharpen_band(sh, d, 960, 540, 0, 540)
    torch.cuda.synchronize()
    ref, S_ref, _ = oracle.sharpen(img, *DEFAULT)
    assert int(s.item()) == S_ref and np.array_equal(out.cpu().numpy(), ref)
    assert halo_rows(540, 0, 540) == (0, 540)


def test_band_errors(sh):
    d = torch.zeros((40, 64), dtype=torch.uint8, device="cuda")
    o = torch.zeros((8, 64), dtype=torch.uint8, device="cuda")
    s = torch.zeros(1, dtype=torch.int64, device="cuda")
    with pytest.raises(SharpError) as e:
        sh.band_edge_sum(d, 64, 40, 2, 10, s)  # row0 not a multiple of 4
    assert e.value.code == SHARP_EINVAL
    with pytest.raises(SharpError) as e:
        sh.band_edge_sum(d, 64, 40, 8, 8, s)  # empty band
    assert e.value.code == SHARP_EINVAL
    with pytest.raises(SharpError) as e:
        sh.band_sharpen(d.cpu(), 64, 40, 0, 8, s, o)  # host pointer
    assert e.value.code == SHARP_EINVAL
    d2 = torch.zeros((40, 68), dtype=torch.uint8, device="cuda")
    with pytest.raises(SharpError) as e:
        sh.band_edge_sum(d2, 68, 40, 0, 8, s)  # W % 16 != 0: no TMA path
    assert e.value.code == SHARP_EUNSUPPORTED
