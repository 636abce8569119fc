"""Seeded synthetic 8-bit frames (see synth.c and DESIGN.md sec. 4).

Shared by the oracle side and the CUDA side of the tests and by bench.py; it
contains none of the sharpening arithmetic.
"""
import ctypes
import os

import numpy as np

KINDS = {"natural": 0, "noise": 1, "ramp": 2, "const": 3, "checker": 4, "impulse": 5}
BASE_SEED = 0x5EED2015  # base seed + config index (+ frame)

_here = os.path.dirname(os.path.abspath(__file__))
_lib = None


def _load():
    global _lib
    if _lib is None:
        path = os.path.join(_here, "libsynth.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(path)
        lib.synth_frames.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                     ctypes.c_int, ctypes.c_uint64, ctypes.c_int, ctypes.c_int]
        lib.synth_frames.restype = ctypes.c_int
        _lib = lib
    return _lib


def frames(n, width, height, kind="natural", seed=BASE_SEED, param=0, threads=0, out=None):
    """Return (or fill `out` with) an [n, height, width] uint8 array.

    Frame f is generated from seed + f.  `out` may be any C-contiguous uint8
    numpy array of that shape (e.g. a view of pinned host memory)."""
    k = KINDS[kind] if isinstance(kind, str) else int(kind)
    if out is None:
        out = np.empty((n, height, width), dtype=np.uint8)
    assert out.dtype == np.uint8 and out.flags["C_CONTIGUOUS"] and out.size == n * width * height
    rc = _load().synth_frames(out.ctypes.data, n, width, height, k, seed, param, threads)
    if rc != 0:
        raise ValueError("synth_frames: bad arguments")
    return out


def image(width, height, kind="natural", seed=BASE_SEED, param=0):
    """One [height, width] uint8 frame."""
    return frames(1, width, height, kind, seed, param)[0]
