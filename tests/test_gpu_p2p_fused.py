"""One fused launch per band (sharp_band_p2p_sharpen): pass 1, the
cross-band all-reduce of the pEdge partials through peer memory (inside the
persistent step kernel) and pass 2, after the peer-memory halo push.  Several
bands of one image on one GPU (each its own context, stream and capped
persistent grid, so all bands co-reside); assembled bands bit-exact vs the
whole-image oracle over epochs, mixed with the four-launch path (same epoch
protocol), and every band's S equal to the image's S."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_EINVAL, SharpError, Sharpener, sharp_band_p2p_sharpen,
                                            sharp_p2p_window_create, sharp_p2p_window_destroy)
from paper_conf_icpp_fanjzac15_b200.bands import P2PBand, band_rows

pytestmark = pytest.mark.gpu
DEFAULT = (1.0, 0.5, 0.5, 2.0)


class Bands:
    def __init__(self, w, h, G):
        self.w, self.h, self.G = w, h, G
        sms = torch.cuda.get_device_properties(0).multi_processor_count
        self.cap = max(1, (2 * sms) // G)  # leave room for the single-CTA halo kernels
        self.cap1 = max(1, (3 * sms) // G)  # one launch per band: all bands' grids co-reside
        self.streams = [torch.cuda.Stream() for _ in range(G)]
        self.sh = [Sharpener() for _ in range(G)]
        for s, st in zip(self.sh, self.streams):
            s.set_stream(st)
        rows = [band_rows(h, G, g) for g in range(G)]
        self.windows = [sharp_p2p_window_create(w, r1 - r0) for r0, r1 in rows]
        self.bands = [P2PBand(self.sh[g], w, h, rank=g, world=G, window=self.windows[g], windows=self.windows)
                      for g in range(G)]
        for b in self.bands:  # every context's scratch now (allocation may synchronise)
            tmp = torch.zeros(1, dtype=torch.int64, device="cuda")
            b.sh.band_edge_sum(b.band, w, h, b.row0, b.row1, tmp)
        torch.cuda.synchronize()

    def run(self, img, epoch, fused=True, prm=DEFAULT, one_launch=False):
        outs = []
        d = torch.from_numpy(img).cuda()
        torch.cuda.synchronize()
        for b, st in zip(self.bands, self.streams):
            with torch.cuda.stream(st):
                b.own.copy_(d[b.row0:b.row1])
                o = torch.full((b.rows_own, self.w), 7, dtype=torch.uint8, device="cuda")
                if one_launch:
                    b.step_one_launch(epoch, o, prm, grid_cap=self.cap1)
                elif fused:
                    b.step_fused(epoch, o, prm, grid_cap=self.cap)
                else:
                    b.step(epoch, o, prm)
                outs.append(o)
        torch.cuda.synchronize()
        out = torch.cat(outs).cpu().numpy()
        sums = [b.sh.batch_sums(1)[0] if (fused or one_launch) else int(b.total.item()) for b in self.bands]
        return out, sums

    def close(self):
        for b in self.bands:
            b.close()
        for p in self.windows:
            sharp_p2p_window_destroy(p)
        for s in self.sh:
            s.close()


@pytest.mark.parametrize("W,H,G", [(1920, 1080, 2), (1920, 1080, 3), (3840, 2160, 4), (256, 64, 8), (960, 40, 5)])
def test_fused_bands_equal_whole_image_over_epochs(W, H, G):
    bands = Bands(W, H, G)
    try:
        plan = [("natural", 1, True), ("noise", 2, True), ("natural", 3, False), ("natural", 4, True)]
        for epoch, (kind, seed, fused) in enumerate(plan, start=1):
            img = synth.image(W, H, kind, seed=synth.BASE_SEED + 100 * G + seed)
            out, sums = bands.run(img, epoch, fused)
            ref, S, _ = oracle.sharpen(img, *DEFAULT)
            assert sums == [S] * G, (epoch, sums, S)
            bad = np.argwhere(out != ref)
            assert bad.size == 0, f"epoch {epoch} fused={fused}: {len(bad)} mismatches, first {bad[:5].tolist()}"
    finally:
        bands.close()


def test_fused_single_band_is_the_whole_image():
    bands = Bands(512, 512, 1)
    try:
        img = synth.image(512, 512, "natural", seed=5)
        out, sums = bands.run(img, 1)
        ref, S, _ = oracle.sharpen(img, *DEFAULT)
        assert sums == [S]
        np.testing.assert_array_equal(out, ref)
    finally:
        bands.close()


def test_fused_rejections():
    with Sharpener() as s:
        win = sharp_p2p_window_create(64, 8)
        o = torch.empty((8, 64), dtype=torch.uint8, device="cuda")
        try:
            for kw in [dict(epoch=0), dict(rank=1), dict(row0=2)]:
                args = dict(windows=[win], rank=0, w=64, h=8, row0=0, row1=8, epoch=1)
                args.update(kw)
                with pytest.raises(SharpError) as e:
                    sharp_band_p2p_sharpen(s.ctx, args["windows"], args["rank"], args["w"], args["h"], args["row0"],
                                           args["row1"], args["epoch"], None, o)
                assert e.value.code == SHARP_EINVAL
        finally:
            sharp_p2p_window_destroy(win)


@pytest.mark.parametrize("W,H,G", [(1920, 1080, 2), (1920, 1080, 3), (3840, 2160, 4), (256, 64, 8), (960, 40, 5)])
def test_one_launch_per_band_equal_whole_image_over_epochs(W, H, G):
    """sharp_band_p2p_step: the halo push folded into the fused launch too --
    one launch per band per image; mixed over epochs with the separate-kernel
    paths (same window protocol)."""
    bands = Bands(W, H, G)
    try:
        plan = [("natural", 1, "one"), ("noise", 2, "one"), ("natural", 3, "fused"), ("natural", 4, "p2p"),
                ("noise", 5, "one")]
        for epoch, (kind, seed, how) in enumerate(plan, start=1):
            img = synth.image(W, H, kind, seed=synth.BASE_SEED + 100 * G + seed)
            out, sums = bands.run(img, epoch, fused=(how == "fused"), one_launch=(how == "one"))
            ref, S, _ = oracle.sharpen(img, *DEFAULT)
            assert sums == [S] * G, (epoch, how, sums, S)
            bad = np.argwhere(out != ref)
            assert bad.size == 0, f"epoch {epoch} {how}: {len(bad)} mismatches, first {bad[:5].tolist()}"
    finally:
        bands.close()
