"""The C ABI from plain C: tests/c_abi_check.c (device and host calls, a
batch, sharp_run_ex with a pitched ROI and a reading switch, the error
contract), every output compared byte for byte with the CPU oracle."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def test_c_program_through_the_abi():
    exe = os.path.join(ROOT, "tests", "c_abi_check")
    if not os.path.exists(exe):
        subprocess.run(["make", "-C", ROOT, "-s", "tests/c_abi_check"], check=True)
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr + r.stdout
    assert "c_abi_check ok" in r.stdout
