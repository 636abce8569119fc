"""CPU checks of bench.py's contract logic (no GPU): the workload description
for weak / strong scaling, the reference arm's line, the NUMA cpulist
parsing.  The timed paths themselves need a B200 (driver runs)."""
import argparse
import importlib.util
import json
import os
import subprocess

import pytest
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def load_bench():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_workload_config_weak_and_strong():
    b = load_bench()
    a = argparse.Namespace(frames=1024, width=1920, height=1080, scaling="weak")
    w = b.workload_config(a, 8)
    assert w["frames"] == 8 * 1024 and w["frames_per_gpu"] == 1024 and "per GPU" in w["workload"]
    a.scaling = "strong"
    st = b.workload_config(a, 8)
    assert st["frames"] == 1024 and st["frames_per_gpu"] is None and "split over 8" in st["parallelism"]
    a.scaling = "weak"
    assert b.workload_config(a, 1)["frames"] == b.workload_config(argparse.Namespace(
        frames=1024, width=1920, height=1080, scaling="strong"), 1)["frames"]


def test_reference_arm_line_on_cpu():
    """--impl reference runs the oracle on host cores (no GPU) and prints the
    contract's line with impl, cpu_baseline and a zero-transfer e2e."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "0", "--ref-sample", "2", "--width", "256", "--height", "128", "--frames", "8"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["unit"] == "Mpix/s" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["e2e"]["h2d_bytes_per_step"] == 0
    assert line["scaling"] == "weak" and line["higher_is_better"] is True


def test_numa_binding_is_best_effort_without_a_gpu():
    b = load_bench()

    class NoGpu:
        class cuda:
            @staticmethod
            def get_device_properties(i):
                raise AttributeError("no GPU")

    assert b.bind_to_gpu_numa_node(NoGpu, 0) is None


def test_gpus_n_self_launches_n_ranks():
    """`bench.py --gpus 2` without torchrun re-launches itself as 2 ranks
    (torch.distributed.run on 127.0.0.1); rank 0 prints ONE line with
    n_gpus == 2 (the reference arm, which runs on host cores, exercises the
    launch without a GPU)."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                        "--steps", "1", "--warmup", "0", "--ref-sample", "2", "--width", "256", "--height", "128",
                        "--frames", "8"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(x) for x in r.stdout.strip().splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout
    assert lines[0]["n_gpus"] == 2 and lines[0]["impl"] == "reference"


def test_gpus_n_beyond_visible_fails_loudly():
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--steps", "1"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT, env=env)
    assert r.returncode != 0 and "visible" in r.stderr


def test_committed_profile_is_keyed_on_the_kernel_sources(monkeypatch):
    """bench.py reports ncu-derived traffic / instruction counts only from a
    capture of the CURRENT kernel sources (profiles/*/traffic*.json carry the
    sources' sha256); a stale capture yields None, never old numbers."""
    b = load_bench()
    cur = b.committed_profile("step")
    if cur is not None:
        assert cur["source_sha256"] == b.kernel_source_hash("step")
        assert b.traffic_per_launch(1000.0) == pytest.approx(1000.0 * cur["dram_bytes_per_px"])
    monkeypatch.setattr(b, "kernel_source_hash", lambda kind: "0" * 64)
    assert b.committed_profile("step") is None
    assert b.traffic_per_launch(1000.0) is None and b.issue_profile() is None
