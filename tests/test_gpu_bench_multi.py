"""bench.py --gpus 2 on a one-GPU box (the SHARP_BENCH_SHARE_GPU hook maps both
ranks onto device 0, gloo plumbing): it self-launches two ranks under
torch.distributed.run and rank 0 prints ONE line with n_gpus == 2, the weak
value over both ranks' frames and the strong-scaling line beside it."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_gpus_2_self_launch():
    env = dict(os.environ, SHARP_BENCH_SHARE_GPU="1")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3",
                        "--frames", "16", "--e2e-steps", "1", "--no-cpu"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(x) for x in r.stdout.strip().splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = lines[0]
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["config"]["frames"] == 32
    assert d["strong_scaling"]["scaling"] == "strong" and d["strong_scaling"]["frames_per_gpu"] == 8
    assert d["value"] > 0 and d["e2e"]["value"] > 0


@pytest.mark.parametrize("exchange", ["nccl", "one"])
def test_bench_bands_2_ranks_share_gpu(exchange):
    """The row-band workload over 2 ranks on one GPU: NCCL send/recv (gloo under
    the share hook) or the one-launch peer-memory path (CUDA IPC windows,
    bounded persistent grids); bit-exact parity is part of the line."""
    env = dict(os.environ, SHARP_BENCH_SHARE_GPU="1")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--workload", "bands",
                        "--exchange", exchange, "--width", "1920", "--height", "1088", "--steps", "3", "--warmup", "2",
                        "--e2e-steps", "1"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(x) for x in r.stdout.strip().splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = lines[0]
    assert d["n_gpus"] == 2 and d["config"]["bands"] == 2
    assert d["parity"]["mismatched_pixels"] == 0
