import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
TESTS = os.path.dirname(os.path.abspath(__file__))
if TESTS not in sys.path:
    sys.path.insert(0, TESTS)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the built libsharp.so")
    config.addinivalue_line("markers", "slow: long-running (full-size parity)")


def _built():
    import subprocess

    # Build the in-tree native artefacts once per session if any is missing
    # (the CPU suite needs liboracle.so / libsynth.so / libsharp.so).
    need = ["oracle/liboracle.so", "synth/libsynth.so",
            "paper_conf_icpp_fanjzac15_b200/libsharp.so"]
    if not all(os.path.exists(os.path.join(ROOT, p)) for p in need):
        subprocess.run(["make", "-C", ROOT, "-s"], check=True)


_built()


@pytest.fixture(scope="session")
def has_gpu():
    import torch

    return torch.cuda.is_available()
