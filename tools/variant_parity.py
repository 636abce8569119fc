#!/usr/bin/env python
"""Bit-exact parity of prebuilt libsharp.so variants against the oracle on the
step-kernel path (ragged tiles, ring rows / columns, partial CTA tiles, lag
rounds).  Each library is copied over the in-tree libsharp.so and checked in
a fresh process.

usage: tools/variant_parity.py build/variants/a.so [b.so ...]
"""
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_icpp_fanjzac15_b200", "libsharp.so")

CASES = [(3, 1920, 1080), (1, 3840, 2160), (2, 1008, 36), (1, 16, 8), (1, 32, 12), (5, 976, 20),
         (40, 1920, 1080), (1, 1936, 1084), (2, 2000, 24)]

CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, ".")
import oracle, synth
from paper_conf_icpp_fanjzac15_b200 import Sharpener
prm = (1.0, 0.5, 0.5, 2.0)
bad = 0
with Sharpener(device=0) as sh:
    sh.set_path(int(os.environ.get("VP_PATH", "1")))
    for (n, W, H) in CASES:
        imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 7 + W + H)
        d = torch.from_numpy(imgs).cuda()
        o = torch.empty_like(d)
        sh.run_batch(d, prm, o)
        torch.cuda.synchronize()
        ref = oracle.sharpen_batch(imgs, *prm)[0]
        m = int((o.cpu().numpy() != ref).sum())
        bad += m
        print(f"  {n} x {W}x{H}: {m} mismatches")
print("PARITY", "OK" if bad == 0 else "FAIL")
'''


def main():
    shutil.copy(LIB, "/tmp/libsharp.orig.so")
    try:
        for v in sys.argv[1:]:
            shutil.copy(v, LIB)
            print(os.path.basename(v), flush=True)
            subprocess.run([sys.executable, "-c", f"CASES = {CASES!r}\n" + CHILD], cwd=ROOT, timeout=600)
    finally:
        shutil.copy("/tmp/libsharp.orig.so", LIB)


if __name__ == "__main__":
    main()
