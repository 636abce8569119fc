"""World-size-2 gloo tests of the N>1 path on CPU (task rule 5): the frame
partition covers every frame exactly once, per-rank results assemble into the
single-rank result, and the timing reduction is the max over ranks.  The
per-frame work here is the CPU oracle standing in for the device kernels (test
infrastructure only); the partition and reduction code is the product's
(paper_conf_icpp_fanjzac15_b200/shard.py), shared with bench.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_fanjzac15_b200.shard import frame_range, max_over_ranks


@pytest.mark.parametrize("n,world", [(1024, 1), (1024, 2), (1024, 8), (7, 2), (3, 4), (0, 2)])
def test_frame_range_partitions_exactly(n, world):
    seen = []
    for r in range(world):
        s, c = frame_range(n, world, r)
        seen.extend(range(s, s + c))
    assert seen == list(range(n))
    counts = [frame_range(n, world, r)[1] for r in range(world)]
    assert max(counts) - min(counts) <= 1


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_dir):
    import oracle
    import synth

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, W, H = 6, 48, 32
    start, cnt = frame_range(n, world, rank)
    imgs = synth.frames(n, W, H, "natural", seed=77)[start:start + cnt]
    outs, sums = oracle.sharpen_batch(imgs, threads=1)
    np.save(os.path.join(out_dir, f"out{rank}.npy"), outs)
    np.save(os.path.join(out_dir, f"sums{rank}.npy"), sums)
    t = max_over_ranks(1.0 + rank)  # each rank "measured" 1+rank ms
    with open(os.path.join(out_dir, f"max{rank}.txt"), "w") as f:
        f.write(repr(t))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_frame_split_equals_single_rank(tmp_path):
    import oracle
    import synth

    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    outs = np.concatenate([np.load(tmp_path / f"out{r}.npy") for r in range(world)])
    sums = np.concatenate([np.load(tmp_path / f"sums{r}.npy") for r in range(world)])
    ref, ref_sums = oracle.sharpen_batch(synth.frames(6, 48, 32, "natural", seed=77), threads=1)
    np.testing.assert_array_equal(outs, ref)
    np.testing.assert_array_equal(sums, ref_sums)
    for r in range(world):
        assert float((tmp_path / f"max{r}.txt").read_text()) == 2.0  # max over ranks


def test_max_over_ranks_identity_without_process_group():
    assert not dist.is_initialized()
    assert max_over_ranks(3.5) == 3.5
