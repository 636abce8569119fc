"""Fused peer-memory band exchange on one GPU.

Several bands of one image, each with its own context and stream, exchange
their halo rows and pEdge partials through each other's windows with the
epoch handshake of bands_p2p.cu (on one device the "peer mappings" are the
other bands' plain device addresses; across GPUs they are CUDA-IPC mappings
over NVLink -- the same kernels).  The assembled bands must equal the
whole-image oracle bit for bit, image after image (epochs), and every band's
all-reduced S must equal the image's S."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_EINVAL, SharpError, Sharpener, sharp_p2p_window_bytes,
                                            sharp_p2p_window_create, sharp_p2p_window_destroy)
from paper_conf_icpp_fanjzac15_b200.bands import P2PBand

pytestmark = pytest.mark.gpu

DEFAULT = (1.0, 0.5, 0.5, 2.0)


class Bands:
    def __init__(self, w, h, G):
        self.w, self.h, self.G = w, h, G
        self.streams = [torch.cuda.Stream() for _ in range(G)]
        self.sh = [Sharpener() for _ in range(G)]
        for s, st in zip(self.sh, self.streams):
            s.set_stream(st)
        from paper_conf_icpp_fanjzac15_b200.bands import band_rows
        rows = [band_rows(h, G, g) for g in range(G)]
        self.windows = [sharp_p2p_window_create(w, r1 - r0) for r0, r1 in rows]
        self.bands = [P2PBand(self.sh[g], w, h, rank=g, world=G, window=self.windows[g], windows=self.windows)
                      for g in range(G)]
        # allocate every context's scratch now (the first band call may synchronise its stream)
        for b in self.bands:
            tmp = torch.zeros(1, dtype=torch.int64, device="cuda")
            b.sh.band_edge_sum(b.band, w, h, b.row0, b.row1, tmp)
        torch.cuda.synchronize()

    def run(self, img, epoch, prm=DEFAULT):
        outs = []
        d = torch.from_numpy(img).cuda()
        torch.cuda.synchronize()
        for b, st in zip(self.bands, self.streams):
            with torch.cuda.stream(st):
                b.own.copy_(d[b.row0:b.row1])
                o = torch.full((b.rows_own, self.w), 7, dtype=torch.uint8, device="cuda")
                b.step(epoch, o, prm)
                outs.append(o)
        torch.cuda.synchronize()
        out = torch.cat(outs).cpu().numpy()
        totals = [int(b.total.item()) for b in self.bands]
        return out, totals

    def close(self):
        for b in self.bands:
            b.close()
        for p in self.windows:
            sharp_p2p_window_destroy(p)
        for s in self.sh:
            s.close()


@pytest.mark.parametrize("W,H,G", [(1920, 1080, 2), (1920, 1080, 3), (3840, 2160, 4), (256, 64, 8), (960, 40, 5)])
def test_p2p_bands_equal_whole_image_over_epochs(W, H, G):
    bands = Bands(W, H, G)
    try:
        for epoch, (kind, seed) in enumerate([("natural", 1), ("noise", 2), ("natural", 3)], start=1):
            img = synth.image(W, H, kind, seed=synth.BASE_SEED + 100 * G + seed)
            out, totals = bands.run(img, epoch)
            ref, S, _ = oracle.sharpen(img, *DEFAULT)
            assert totals == [S] * G, (totals, S)
            bad = np.argwhere(out != ref)
            assert bad.size == 0, f"epoch {epoch}: {len(bad)} mismatches, first {bad[:5].tolist()}"
    finally:
        bands.close()


def test_p2p_single_band_is_the_whole_image():
    bands = Bands(512, 512, 1)
    try:
        img = synth.image(512, 512, "natural", seed=5)
        out, totals = bands.run(img, 1)
        ref, S, _ = oracle.sharpen(img, *DEFAULT)
        assert totals == [S]
        np.testing.assert_array_equal(out, ref)
    finally:
        bands.close()


def test_p2p_window_geometry_and_rejections():
    assert sharp_p2p_window_bytes(1920, 540) == 1024 + (540 + 8) * 1920
    assert sharp_p2p_window_bytes(1921, 540) == 0  # w % 16
    assert sharp_p2p_window_bytes(1920, 3) == 0    # fewer than 4 rows
    with Sharpener() as s:
        from paper_conf_icpp_fanjzac15_b200 import sharp_band_p2p_allreduce, sharp_band_p2p_halo
        win = sharp_p2p_window_create(64, 8)
        try:
            with pytest.raises(SharpError) as e:
                sharp_band_p2p_halo(s.ctx, win, 64, 8, None, 0, None, 0)  # epoch 0
            assert e.value.code == SHARP_EINVAL
            p = torch.zeros(1, dtype=torch.int64, device="cuda")
            with pytest.raises(SharpError) as e:
                sharp_band_p2p_allreduce(s.ctx, [win], 1, p, 1, p)  # rank >= n_ranks
            assert e.value.code == SHARP_EINVAL
        finally:
            sharp_p2p_window_destroy(win)
