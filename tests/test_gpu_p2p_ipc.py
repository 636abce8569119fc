"""The multi-process half of the fused peer-memory band exchange (SURVEY.md
sec. 8(f) NEXT 2): 2 and 3 processes, one band each, whose
windows are exchanged as CUDA IPC handles over gloo (bands.P2PBand
multi-process mode) -- the halo rows and the L174 pEdge partials then cross
ADDRESS SPACES through the mapped windows, with the epoch-flag protocol.  On a
one-GPU box all ranks share device 0 (cudaIpcOpenMemHandle maps another
process's allocation on the same device); the four-launch path, the fused
launch and the one-launch path run over six epochs, every band bit-exact vs
the oracle and every rank's S equal to the image's S."""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    with socket.socket(socket.AF_INET, socket.SOCK_STREAM) as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world,WH", [(2, (1920, 1080)), (3, (960, 544))])
def test_ipc_windows_across_processes(world, WH):
    port = free_port()
    procs = []
    for r in range(world):
        env = dict(os.environ, RANK=str(r), WORLD_SIZE=str(world), MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port),
                   LOCAL_RANK=str(r))
        procs.append(subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "_p2p_ipc_worker.py"),
                                       str(WH[0]), str(WH[1])], env=env, stdout=subprocess.PIPE,
                                      stderr=subprocess.STDOUT, text=True))
    outs = []
    try:
        for p in procs:
            out, _ = p.communicate(timeout=240)
            outs.append(out)
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    for r, (p, out) in enumerate(zip(procs, outs)):
        assert p.returncode == 0, f"rank {r} failed:\n{out[-3000:]}"
