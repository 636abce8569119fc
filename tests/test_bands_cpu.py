"""Row-band sharding host logic on CPU (task rule 5): the band partition, the
4-row halo (necessary and sufficient, checked on the oracle's stages), the
C ABI's sharp_band_halo (host-only, no GPU needed), and the world-size-2/3
gloo plumbing of bands.py (halo exchange by send/recv, all-reduce of the
per-band pEdge sums).  The per-band compute here is the CPU oracle standing
in for the device kernels (test infrastructure only)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import sharp_band_halo
from paper_conf_icpp_fanjzac15_b200.bands import HALO, band_rows, exchange_halos, halo_rows


@pytest.mark.parametrize("h,world", [(1080, 1), (1080, 2), (1080, 8), (4320, 8), (16384, 8), (40, 10), (8, 2),
                                     (1084, 3)])
def test_band_rows_partition(h, world):
    rows = [band_rows(h, world, g) for g in range(world)]
    assert rows[0][0] == 0 and rows[-1][1] == h
    for (a0, a1), (b0, _) in zip(rows, rows[1:]):
        assert a1 == b0
    assert all(r0 % 4 == 0 and r1 % 4 == 0 and r1 > r0 for r0, r1 in rows)
    sizes = [r1 - r0 for r0, r1 in rows]
    assert max(sizes) - min(sizes) <= 4


def test_band_rows_rejects():
    for args in [(1082, 2, 0), (8, 3, 0), (1080, 2, 2), (4, 1, 0)]:
        with pytest.raises(ValueError):
            band_rows(*args)


@pytest.mark.parametrize("h,r0,r1", [(1080, 0, 540), (1080, 540, 1080), (1080, 4, 8), (8, 0, 8), (4320, 1080, 2160)])
def test_halo_rows_match_c_abi(h, r0, r1):
    assert sharp_band_halo(h, r0, r1) == halo_rows(h, r0, r1)


@pytest.mark.parametrize("args", [(1080, 2, 8), (1080, 8, 8), (1080, 0, 1084), (1082, 0, 8), (1080, -4, 8)])
def test_halo_rows_c_abi_rejects(args):
    from paper_conf_icpp_fanjzac15_b200 import SharpError
    with pytest.raises(SharpError):
        sharp_band_halo(*args)


def _stage_rows(img, r0, r1):
    """The per-pixel inputs of the final steps on rows [r0, r1): U (L140-L146),
    pEdge (L158-L172) and the 3x3 max/min of O (L182)."""
    H, W = img.shape
    U = oracle.upscale(oracle.downscale(img), W, H)
    pE = oracle.sobel(img)
    pad = np.pad(img.astype(np.int32), 1, mode="edge")
    win = np.stack([pad[1 + dy:1 + dy + H, 1 + dx:1 + dx + W] for dy in (-1, 0, 1) for dx in (-1, 0, 1)])
    return U[r0:r1], pE[r0:r1], win.max(0)[r0:r1], win.min(0)[r0:r1]


@pytest.mark.parametrize("r0,r1", [(8, 16), (12, 28), (20, 40), (4, 8)])
def test_four_halo_rows_suffice(r0, r1):
    """Changing every image row outside [r0-4, r1+4) leaves U, pEdge and the
    overshoot window of rows [r0, r1) unchanged (so with the all-reduced S the
    band's output is the whole image's)."""
    H, W = 48, 40
    img = synth.image(W, H, "noise", seed=r0 * 100 + r1)
    in0, in1 = halo_rows(H, r0, r1)
    other = img.copy()
    rng = np.random.default_rng(1)
    other[:in0] = rng.integers(0, 256, other[:in0].shape, dtype=np.uint8)
    other[in1:] = rng.integers(0, 256, other[in1:].shape, dtype=np.uint8)
    for a, b in zip(_stage_rows(img, r0, r1), _stage_rows(other, r0, r1)):
        np.testing.assert_array_equal(a, b)


def test_three_halo_rows_do_not_suffice():
    """Row r0-4 feeds D row r0/4-1, which the upscale of row r0 reads (L146)."""
    H, W, r0, r1 = 48, 40, 16, 32
    img = synth.image(W, H, "noise", seed=4)
    other = img.copy()
    other[r0 - HALO] = 255 - other[r0 - HALO]
    U0, _, _, _ = _stage_rows(img, r0, r1)
    U1, _, _, _ = _stage_rows(other, r0, r1)
    assert not np.array_equal(U0, U1)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    W, H = 40, 44
    img = synth.image(W, H, "natural", seed=21)
    r0, r1 = band_rows(H, world, rank)
    own = torch.from_numpy(img[r0:r1].copy())           # this rank holds only its rows
    band = exchange_halos(own, H, r0, r1)               # + halo rows from the neighbours
    in0, in1 = halo_rows(H, r0, r1)
    np.save(os.path.join(out_dir, f"band{rank}.npy"), band.numpy())
    # stand-in for sharp_band_edge_sum: the oracle's pEdge of the rows this rank owns
    part = torch.tensor([int(oracle.sobel(img)[r0:r1].astype(np.int64).sum())], dtype=torch.int64)
    dist.all_reduce(part, op=dist.ReduceOp.SUM)
    with open(os.path.join(out_dir, f"S{rank}.txt"), "w") as f:
        f.write(f"{in0} {in1} {int(part.item())}")
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_halo_exchange_and_allreduce(tmp_path, world):
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    img = synth.image(40, 44, "natural", seed=21)
    S_ref, _ = oracle.reduce(oracle.sobel(img))
    for r in range(world):
        in0, in1, S = map(int, (tmp_path / f"S{r}.txt").read_text().split())
        np.testing.assert_array_equal(np.load(tmp_path / f"band{r}.npy"), img[in0:in1])
        assert S == S_ref
