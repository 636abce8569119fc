"""Worker of tests/test_gpu_p2p_ipc.py: one rank of a row-band-sharded image
on its own process, windows exchanged as CUDA IPC handles over gloo
(bands.P2PBand multi-process mode).  Every rank checks its band against the
oracle for every epoch and exits 0 on success."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_fanjzac15_b200 import Sharpener  # noqa: E402
from paper_conf_icpp_fanjzac15_b200.bands import P2PBand  # noqa: E402


def main():
    W, H = int(sys.argv[1]), int(sys.argv[2])
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(rank % torch.cuda.device_count())
    st = torch.cuda.Stream()
    torch.cuda.set_stream(st)
    sh = Sharpener(device=torch.cuda.current_device())
    sh.set_stream(st)
    p2p = P2PBand(sh, W, H)  # IPC handle exchange over gloo
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    cap = max(1, (2 * sms) // world)  # ranks sharing one GPU: bounded persistent grids
    prm = (1.3, 0.5, 0.5, 2.0)
    modes = ["step", "fused", "one", "one", "fused", "step"]
    bad = 0
    for e, mode in enumerate(modes, start=1):
        img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 100 + e)
        p2p.own.copy_(torch.from_numpy(img[p2p.row0:p2p.row1].copy()).cuda())
        torch.cuda.synchronize()
        dist.barrier()  # every rank's rows are in its window before any halo push
        out = torch.empty((p2p.rows_own, W), dtype=torch.uint8, device="cuda")
        if mode == "step":
            p2p.step(e, out, prm)
        elif mode == "fused":
            p2p.step_fused(e, out, prm, grid_cap=cap)
        else:
            p2p.step_one_launch(e, out, prm, grid_cap=cap)
        torch.cuda.synchronize()
        ref, S, _ = oracle.sharpen(img, *prm)
        n = int((out.cpu().numpy() != ref[p2p.row0:p2p.row1]).sum())
        S_band = int(p2p.total.item()) if mode == "step" else int(sh.batch_sums(1)[0])
        if n or S_band != S:
            print(f"rank {rank} epoch {e} ({mode}): {n} mismatched pixels, S {S_band} vs {S}", flush=True)
            bad += 1
        dist.barrier()  # the next epoch's rows are written only after every rank read this one's halos
    p2p.close()
    sh.close()
    dist.destroy_process_group()
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
