"""ctypes wrapper of the CPU oracle (oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py -- never by the product
package paper_conf_icpp_fanjzac15_b200/.
"""
import ctypes
import os

import numpy as np

_here = os.path.dirname(os.path.abspath(__file__))
_lib = None

_P = ctypes.c_void_p
_I = ctypes.c_int
_F = ctypes.c_float
_D = ctypes.c_double


def _load():
    global _lib
    if _lib is None:
        path = os.path.join(_here, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(path)
        sigs = {
            "oracle_check_geometry": ([_I, _I], _I),
            "oracle_downscale": ([_P, _I, _I, _P], None),
            "oracle_upscale": ([_P, _I, _I, _P], None),
            "oracle_upscale_steps": ([_P, _I, _I, _P, _I], None),
            "oracle_perror": ([_P, _P, _I, _P], None),
            "oracle_sobel": ([_P, _I, _I, _P], None),
            "oracle_reduce": ([_P, _I, _I, _P, _P], None),
            "oracle_strength": ([_P, _I, _D, _F, _F, _P], None),
            "oracle_preliminary": ([_P, _P, _P, _I, _P], None),
            "oracle_overshoot": ([_P, _P, _P, _I, _I, _D, _F, _F, _P], None),
            "oracle_output": ([_P, _I, _P], None),
            "oracle_sharpen": ([_P, _I, _I, _F, _F, _F, _F, _P, _P, _P], _I),
            "oracle_sharpen_batch": ([_P, _I, _I, _I, _F, _F, _F, _F, _P, _P, _I], _I),
            "oracle_downscale_ex": ([_P, _I, _I, _I, _P], None),
            "oracle_upscale_ex": ([_P, _I, _I, _I, _P], None),
            "oracle_upscale_steps_ex": ([_P, _I, _I, _P, _I, _I], None),
            "oracle_reduce_ex": ([_P, _I, _I, _I, _P, _P], None),
            "oracle_strength_ex": ([_P, _I, _D, _F, _F, _F, _I, _P], None),
            "oracle_overshoot_ex": ([_P, _P, _P, _I, _I, _D, _F, _F, _I, _P], None),
            "oracle_output_ex": ([_P, _I, _I, _P], None),
            "oracle_sharpen_ex": ([_P, _I, _I, _I, _F, _F, _F, _F, _I, _P, _I, _P, _P], _I),
        }
        for name, (args, res) in sigs.items():
            fn = getattr(lib, name)
            fn.argtypes = args
            fn.restype = res
        _lib = lib
    return _lib


DEFAULTS = dict(amount=1.0, gamma=0.5, osc_gain=0.5, osc_scale=2.0)  # DESIGN.md R16


def _c(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a, a.ctypes.data


def downscale(O):
    O, p = _c(O, np.uint8)
    H, W = O.shape
    D = np.empty((H // 4, W // 4), np.float32)
    _load().oracle_downscale(p, W, H, D.ctypes.data)
    return D


def upscale(D, W, H):
    D, p = _c(D, np.float32)
    U = np.empty((H, W), np.float32)
    _load().oracle_upscale(p, W, H, U.ctypes.data)
    return U


def upscale_steps(D, W, H, last_step):
    D, p = _c(D, np.float32)
    U = np.empty((H, W), np.float32)
    _load().oracle_upscale_steps(p, W, H, U.ctypes.data, last_step)
    return U


def perror(O, U):
    O, po = _c(O, np.uint8)
    U, pu = _c(U, np.float32)
    E = np.empty(O.shape, np.float32)
    _load().oracle_perror(po, pu, O.size, E.ctypes.data)
    return E


def sobel(O):
    O, p = _c(O, np.uint8)
    H, W = O.shape
    pE = np.empty((H, W), np.int32)
    _load().oracle_sobel(p, W, H, pE.ctypes.data)
    return pE


def reduce(pE):
    pE, p = _c(pE, np.int32)
    H, W = pE.shape
    S = ctypes.c_uint64()
    mean = ctypes.c_double()
    _load().oracle_reduce(p, W, H, ctypes.byref(S), ctypes.byref(mean))
    return S.value, mean.value


def strength(pE, mean, amount, gamma):
    pE, p = _c(pE, np.int32)
    adj = np.empty(pE.shape, np.float32)
    _load().oracle_strength(p, pE.size, mean, amount, gamma, adj.ctypes.data)
    return adj


def preliminary(adj, E, U):
    adj, pa = _c(adj, np.float32)
    E, pe = _c(E, np.float32)
    U, pu = _c(U, np.float32)
    P = np.empty(adj.shape, np.float32)
    _load().oracle_preliminary(pa, pe, pu, adj.size, P.ctypes.data)
    return P


def overshoot(O, P, pE, mean, osc_gain, osc_scale):
    O, po = _c(O, np.uint8)
    P, pp = _c(P, np.float32)
    pE, pq = _c(pE, np.int32)
    H, W = O.shape
    F = np.empty((H, W), np.float32)
    _load().oracle_overshoot(po, pp, pq, W, H, mean, osc_gain, osc_scale, F.ctypes.data)
    return F


def output(F):
    F, p = _c(F, np.float32)
    out = np.empty(F.shape, np.uint8)
    _load().oracle_output(p, F.size, out.ctypes.data)
    return out


def sharpen(O, amount=1.0, gamma=0.5, osc_gain=0.5, osc_scale=2.0):
    """Whole pipeline -> (out uint8 [H,W], S, mean).  Raises on invalid input."""
    O, p = _c(O, np.uint8)
    H, W = O.shape
    out = np.empty((H, W), np.uint8)
    S = ctypes.c_uint64()
    mean = ctypes.c_double()
    rc = _load().oracle_sharpen(p, W, H, amount, gamma, osc_gain, osc_scale, out.ctypes.data,
                                ctypes.byref(S), ctypes.byref(mean))
    if rc != 0:
        raise ValueError("oracle_sharpen: invalid geometry or parameters")
    return out, S.value, mean.value


def sharpen_batch(imgs, amount=1.0, gamma=0.5, osc_gain=0.5, osc_scale=2.0, threads=0):
    """[n,H,W] -> (outs [n,H,W], sums [n] uint64).  Frames split over threads."""
    imgs, p = _c(imgs, np.uint8)
    n, H, W = imgs.shape
    outs = np.empty_like(imgs)
    sums = np.empty(n, np.uint64)
    rc = _load().oracle_sharpen_batch(p, n, W, H, amount, gamma, osc_gain, osc_scale,
                                      outs.ctypes.data, sums.ctypes.data, threads)
    if rc != 0:
        raise ValueError("oracle_sharpen_batch: invalid geometry or parameters")
    return outs, sums


# ---- reading switches (oracle.h ORACLE_READ_*)
READ_INT_DOWNSCALE = 1   # R2
READ_COLUMN_WINS = 2     # R5
READ_INTERIOR_MEAN = 4   # R8
READ_STRENGTH_EXP = 8    # R9
READ_OSC_CONST = 16      # R11
READ_TRUNCATE = 32       # R14
READ_ALL = 63


def downscale_ex(O, flags):
    O, p = _c(O, np.uint8)
    H, W = O.shape
    D = np.empty((H // 4, W // 4), np.float32)
    _load().oracle_downscale_ex(p, W, H, flags, D.ctypes.data)
    return D


def upscale_ex(D, W, H, flags, last_step=8):
    D, p = _c(D, np.float32)
    U = np.empty((H, W), np.float32)
    _load().oracle_upscale_steps_ex(p, W, H, U.ctypes.data, last_step, flags)
    return U


def reduce_ex(pE, flags):
    pE, p = _c(pE, np.int32)
    H, W = pE.shape
    S = ctypes.c_uint64()
    mean = ctypes.c_double()
    _load().oracle_reduce_ex(p, W, H, flags, ctypes.byref(S), ctypes.byref(mean))
    return S.value, mean.value


def strength_ex(pE, mean, amount, gamma, osc_scale, flags):
    pE, p = _c(pE, np.int32)
    adj = np.empty(pE.shape, np.float32)
    _load().oracle_strength_ex(p, pE.size, mean, amount, gamma, osc_scale, flags, adj.ctypes.data)
    return adj


def overshoot_ex(O, P, pE, mean, osc_gain, osc_scale, flags):
    O, po = _c(O, np.uint8)
    P, pp = _c(P, np.float32)
    pE, pq = _c(pE, np.int32)
    H, W = O.shape
    F = np.empty((H, W), np.float32)
    _load().oracle_overshoot_ex(po, pp, pq, W, H, mean, osc_gain, osc_scale, flags, F.ctypes.data)
    return F


def output_ex(F, flags):
    F, p = _c(F, np.float32)
    out = np.empty(F.shape, np.uint8)
    _load().oracle_output_ex(p, F.size, flags, out.ctypes.data)
    return out


def sharpen_ex(O, amount=1.0, gamma=0.5, osc_gain=0.5, osc_scale=2.0, flags=0):
    """General geometry (R1': any H, W >= 5, replicate-extended to multiples of
    4, sharpened, cropped) with reading switches -> (out [H,W], S, mean).
    O may be a strided 2-D view (rows at any pitch, unit column stride)."""
    O = np.asarray(O, dtype=np.uint8)
    if O.ndim != 2 or O.strides[1] != 1:
        O = np.ascontiguousarray(O)
    H, W = O.shape
    out = np.empty((H, W), np.uint8)
    S = ctypes.c_uint64()
    mean = ctypes.c_double()
    rc = _load().oracle_sharpen_ex(O.ctypes.data, W, H, O.strides[0], amount, gamma, osc_gain, osc_scale, flags,
                                   out.ctypes.data, W, ctypes.byref(S), ctypes.byref(mean))
    if rc != 0:
        raise ValueError("oracle_sharpen_ex: invalid geometry, parameters or flags")
    return out, S.value, mean.value
