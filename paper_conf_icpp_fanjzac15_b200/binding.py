"""ctypes binding of include/sharp.h -- same names as the C ABI.

Marshalling only (pointers, sizes, parameter structs).  The library is loaded
from this package directory (built in-tree by `make`); a missing library is an
error, never a fallback.
"""
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
library_path = os.path.join(_HERE, "libsharp.so")

SHARP_OK = 0
SHARP_EINVAL = -1
SHARP_ENOMEM = -2
SHARP_ECUDA = -3
SHARP_ENCCL = -4
SHARP_EUNSUPPORTED = -5
SHARP_ESTATE = -6
LUT_SIZE = 1536
# kernel paths (sharp_set_path) and stages (sharp_get_stage_times), include/sharp.h
SHARP_PATH_AUTO = 0
SHARP_PATH_STEP = 1
SHARP_PATH_TWO_PASS = 2
SHARP_PATH_STAGED = 3
SHARP_PATH_RES = 4
SHARP_PATH_FUSED = 5
SHARP_PATH_FUSED_EXP = 6
STAGE_NAMES = ("downscale", "border", "center", "sobel", "reduction", "strength", "sharpness")
SHARP_NUM_STAGES = len(STAGE_NAMES)


class SharpParams(ctypes.Structure):
    _fields_ = [("amount", ctypes.c_float), ("gamma", ctypes.c_float),
                ("osc_gain", ctypes.c_float), ("osc_scale", ctypes.c_float)]


class SharpConfig(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("max_width", ctypes.c_int), ("max_height", ctypes.c_int),
                ("max_frames", ctypes.c_int), ("streams", ctypes.c_int), ("chunk_frames", ctypes.c_int),
                ("num_devices", ctypes.c_int), ("device_ids", ctypes.POINTER(ctypes.c_int)), ("shard", ctypes.c_int)]


# multi-device sharding (sharp_config.shard, include/sharp.h)
SHARP_SHARD_AUTO = 0
SHARP_SHARD_NONE = 1
SHARP_SHARD_ROWS = 2
SHARP_SHARD_FRAMES = 3


class SharpStats(ctypes.Structure):
    _fields_ = [("edge_sum", ctypes.c_uint64), ("edge_mean", ctypes.c_double),
                ("device_ms", ctypes.c_float), ("total_ms", ctypes.c_float),
                ("frames", ctypes.c_int), ("kernels", ctypes.c_int)]


class SharpLayout(ctypes.Structure):
    """Byte strides of a batch (include/sharp.h sharp_layout); 0 = dense default."""
    _fields_ = [("pitch", ctypes.c_size_t), ("frame_stride", ctypes.c_size_t), ("elem_stride", ctypes.c_int)]


# reading switches (include/sharp.h SHARP_READ_*)
SHARP_READ_INT_DOWNSCALE = 1   # R2
SHARP_READ_COLUMN_WINS = 2     # R5
SHARP_READ_INTERIOR_MEAN = 4   # R8
SHARP_READ_STRENGTH_EXP = 8    # R9
SHARP_READ_OSC_CONST = 16      # R11
SHARP_READ_TRUNCATE = 32       # R14


class SharpKernelTimes(ctypes.Structure):
    _fields_ = [("pass1_ms", ctypes.c_float), ("pass2_ms", ctypes.c_float),
                ("pass1_launches", ctypes.c_int), ("pass2_launches", ctypes.c_int),
                ("step_ms", ctypes.c_float), ("step_launches", ctypes.c_int),
                ("pixels", ctypes.c_double)]


_P = ctypes.c_void_p
_I = ctypes.c_int
_SIGS = {
    "sharp_create": ([ctypes.POINTER(_P), ctypes.POINTER(SharpConfig)], _I),
    "sharp_destroy": ([_P], None),
    "sharp_default_params": ([ctypes.POINTER(SharpParams)], None),
    "sharp_set_stream": ([_P, _P], _I),
    "sharp_run": ([_P, _P, _I, _I, ctypes.POINTER(SharpParams), _P], _I),
    "sharp_run_batch": ([_P, _P, _I, _I, _I, ctypes.POINTER(SharpParams), _P], _I),
    "sharp_enqueue_batch": ([_P, _P, _I, _I, _I, ctypes.POINTER(SharpParams), _P], _I),
    "sharp_get_stats": ([_P, ctypes.POINTER(SharpStats)], _I),
    "sharp_get_batch_sums": ([_P, _P, _I], _I),
    "sharp_set_profiling": ([_P, _I], _I),
    "sharp_get_kernel_times": ([_P, ctypes.POINTER(SharpKernelTimes)], _I),
    "sharp_strerror": ([_I], ctypes.c_char_p),
    "sharp_last_error": ([_P], ctypes.c_char_p),
    "sharp_version": ([], ctypes.c_char_p),
    "sharp_band_halo": ([_I, _I, _I, ctypes.POINTER(_I), ctypes.POINTER(_I)], _I),
    "sharp_band_edge_sum": ([_P, _P, _I, _I, _I, _I, _P], _I),
    "sharp_band_sharpen": ([_P, _P, _I, _I, _I, _I, _P, ctypes.POINTER(SharpParams), _P], _I),
    "sharp_p2p_window_bytes": ([_I, _I], ctypes.c_size_t),
    "sharp_p2p_window_create": ([_I, _I, ctypes.POINTER(_P)], _I),
    "sharp_p2p_window_destroy": ([_P], None),
    "sharp_band_p2p_halo": ([_P, _P, _I, _I, _P, _I, _P, ctypes.c_uint64], _I),
    "sharp_band_p2p_allreduce": ([_P, ctypes.POINTER(_P), _I, _I, _P, ctypes.c_uint64, _P], _I),
    "sharp_ipc_get_handle": ([_P, _P], _I),
    "sharp_ipc_open_handle": ([_P, ctypes.POINTER(_P)], _I),
    "sharp_ipc_close_handle": ([_P], _I),
    "sharp_set_path": ([_P, _I], _I),
    "sharp_get_path": ([_P], _I),
    "sharp_get_stage_times": ([_P, ctypes.POINTER(ctypes.c_float), _I], _I),
    "sharp_band_p2p_sharpen": ([_P, ctypes.POINTER(_P), _I, _I, _I, _I, _I, _I, ctypes.c_uint64,
                                ctypes.POINTER(SharpParams), _P, _I], _I),
    "sharp_band_p2p_step": ([_P, ctypes.POINTER(_P), _I, _I, _I, _I, _I, _I, _I, ctypes.c_uint64,
                             ctypes.POINTER(SharpParams), _P, _I], _I),
    "sharp_run_ex": ([_P, _P, ctypes.POINTER(SharpLayout), _I, _I, _I, _I, ctypes.POINTER(SharpParams), _I, _P,
                      ctypes.POINTER(SharpLayout)], _I),
    "sharp_band_rows": ([_I, _I, _I, ctypes.POINTER(_I), ctypes.POINTER(_I)], _I),
    "sharp_run_bands": ([_P, ctypes.POINTER(_P), _I, _I, ctypes.POINTER(SharpParams), ctypes.POINTER(_P)], _I),
}

_lib = None


def lib():
    """The loaded libsharp.so (raises if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(library_path):
            raise RuntimeError(f"{library_path} is missing: build it with `make` / __graft_entry__.build(); "
                               "there is no CPU fallback")
        L = ctypes.CDLL(library_path)
        for name, (args, res) in _SIGS.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


class SharpError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{msg} ({code})")
        self.code = code


def _addr(buf):
    """Raw address of a torch tensor / numpy array / int (no copies)."""
    if buf is None:
        return None
    if isinstance(buf, int):
        return buf
    if hasattr(buf, "data_ptr"):  # torch.Tensor
        if not buf.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return buf.data_ptr()
    if hasattr(buf, "ctypes"):  # numpy
        if not buf.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return buf.ctypes.data
    raise TypeError(f"unsupported buffer type {type(buf)}")


def _params(p):
    if p is None:
        return None
    if isinstance(p, SharpParams):
        return p
    if isinstance(p, dict):
        d = sharp_default_params()
        for k, v in p.items():
            setattr(d, k, float(v))
        return d
    return SharpParams(*[float(x) for x in p])


def _check(rc, ctx=None):
    if rc != SHARP_OK:
        detail = sharp_last_error(ctx) if ctx else ""
        raise SharpError(rc, f"{sharp_strerror(rc)}: {detail}")
    return rc


# ---------------------------------------------------------------- C-ABI names
def sharp_create(cfg=None):
    """-> opaque context handle (int).  cfg: SharpConfig or dict or None."""
    keep = None
    if isinstance(cfg, dict):
        c = SharpConfig(device=-1)
        for k, v in cfg.items():
            if k == "device_ids":
                if v:
                    keep = (ctypes.c_int * len(v))(*[int(x) for x in v])
                    c.device_ids = keep
                    c.num_devices = len(v)
                continue
            setattr(c, k, int(v))
        cfg = c
    h = _P()
    rc = lib().sharp_create(ctypes.byref(h), ctypes.byref(cfg) if cfg is not None else None)
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_create: {sharp_strerror(rc)}")
    return h.value


def sharp_destroy(ctx):
    lib().sharp_destroy(ctx)


def sharp_band_rows(h, n_bands, band):
    """Rows [row0, row1) of band `band` of `n_bands` (the h/4 block rows split evenly)."""
    a, b = _I(), _I()
    rc = lib().sharp_band_rows(h, n_bands, band, ctypes.byref(a), ctypes.byref(b))
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_band_rows: {sharp_strerror(rc)}")
    return a.value, b.value


def sharp_run_bands(ctx, bands, w, h, params, outs):
    """bands / outs: per device of the context, device buffers of the band's rows."""
    arr_in = (_P * len(bands))(*[_addr(b) for b in bands])
    arr_out = (_P * len(outs))(*[_addr(o) for o in outs])
    return _check(lib().sharp_run_bands(ctx, arr_in, w, h, _pp(params), arr_out), ctx)


def sharp_default_params():
    p = SharpParams()
    lib().sharp_default_params(ctypes.byref(p))
    return p


def sharp_set_stream(ctx, stream):
    """stream: torch.cuda.Stream, raw cudaStream_t int, or None (context's own).
    torch's default stream has cuda_stream == 0, i.e. the legacy default
    stream: it is passed as cudaStreamLegacy ((void *) 1), because a NULL
    handle means "the context's own stream" in the C ABI."""
    s = getattr(stream, "cuda_stream", stream)
    if hasattr(stream, "cuda_stream") and s == 0:
        s = 1  # cudaStreamLegacy
    return _check(lib().sharp_set_stream(ctx, s), ctx)


def _pp(params):
    p = _params(params)
    return ctypes.byref(p) if p is not None else None


def sharp_run(ctx, img, w, h, params, out):
    return _check(lib().sharp_run(ctx, _addr(img), w, h, _pp(params), _addr(out)), ctx)


def sharp_run_batch(ctx, imgs, n, w, h, params, outs):
    return _check(lib().sharp_run_batch(ctx, _addr(imgs), n, w, h, _pp(params), _addr(outs)), ctx)


def _raw_addr(buf):
    """Address of a (possibly strided) torch tensor / numpy array / int."""
    if isinstance(buf, int):
        return buf
    if hasattr(buf, "data_ptr"):
        return buf.data_ptr()
    if hasattr(buf, "ctypes"):
        return buf.ctypes.data
    raise TypeError(f"unsupported buffer type {type(buf)}")


def _layout(l):
    if l is None or isinstance(l, SharpLayout):
        return l
    if isinstance(l, dict):
        return SharpLayout(**l)
    return SharpLayout(*l)


def sharp_run_ex(ctx, imgs, in_layout, n, channels, w, h, params, flags, outs, out_layout):
    """imgs / outs: base addresses (tensors or arrays: their first element);
    layouts: SharpLayout, dict, tuple (pitch, frame_stride, elem_stride) or None."""
    li, lo = _layout(in_layout), _layout(out_layout)
    return _check(lib().sharp_run_ex(ctx, _raw_addr(imgs), ctypes.byref(li) if li is not None else None, n, channels,
                                     w, h, _pp(params), int(flags), _raw_addr(outs),
                                     ctypes.byref(lo) if lo is not None else None), ctx)


def layout_of(t, channels_last=False):
    """(n, channels, h, w, SharpLayout) of a uint8 tensor / array view:
    [H, W], [N, H, W], or with channels_last=True [H, W, C] / [N, H, W, C]."""
    shape = tuple(t.shape)
    st = tuple(t.stride()) if hasattr(t, "stride") and callable(t.stride) else tuple(t.strides)
    if channels_last:
        if len(shape) == 3:
            shape, st = (1,) + shape, (0,) + st
        n, h, w, c = shape
        fs, pitch, es, cs = st
        if c > 1 and cs != 1:
            raise ValueError("channels must be adjacent bytes (channel stride 1)")
    else:
        if len(shape) == 2:
            shape, st = (1,) + shape, (0,) + st
        n, h, w = shape
        fs, pitch, es = st
        c = 1
    if n == 1:
        fs = 0
    return n, c, h, w, SharpLayout(pitch=pitch, frame_stride=fs, elem_stride=es)


def sharp_enqueue_batch(ctx, d_imgs, n, w, h, params, d_outs):
    return _check(lib().sharp_enqueue_batch(ctx, _addr(d_imgs), n, w, h, _pp(params), _addr(d_outs)), ctx)


def sharp_get_stats(ctx):
    s = SharpStats()
    _check(lib().sharp_get_stats(ctx, ctypes.byref(s)), ctx)
    return s


def sharp_get_batch_sums(ctx, n):
    arr = (ctypes.c_uint64 * n)()
    _check(lib().sharp_get_batch_sums(ctx, ctypes.cast(arr, _P), n), ctx)
    return list(arr)


def sharp_set_profiling(ctx, enable):
    return _check(lib().sharp_set_profiling(ctx, int(bool(enable))), ctx)


def sharp_get_kernel_times(ctx):
    t = SharpKernelTimes()
    _check(lib().sharp_get_kernel_times(ctx, ctypes.byref(t)), ctx)
    return t


SHARP_P2P_CTL_BYTES = 1024
SHARP_IPC_HANDLE_BYTES = 64


def sharp_p2p_window_bytes(w, rows_own):
    return int(lib().sharp_p2p_window_bytes(w, rows_own))


def sharp_p2p_window_create(w, rows_own):
    """-> device address (int) of a zeroed window (caller owns it)."""
    p = _P()
    rc = lib().sharp_p2p_window_create(w, rows_own, ctypes.byref(p))
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_p2p_window_create: {sharp_strerror(rc)}")
    return p.value


def sharp_p2p_window_destroy(d_window):
    lib().sharp_p2p_window_destroy(d_window)


def sharp_band_p2p_halo(ctx, self_window, w, rows_own, up_window, up_rows_own, down_window, epoch):
    return _check(lib().sharp_band_p2p_halo(ctx, self_window, w, rows_own, up_window or None, up_rows_own,
                                            down_window or None, int(epoch)), ctx)


def sharp_band_p2p_allreduce(ctx, windows, rank, d_partial, epoch, d_total):
    arr = (_P * len(windows))(*windows)
    return _check(lib().sharp_band_p2p_allreduce(ctx, arr, len(windows), rank, _addr(d_partial), int(epoch),
                                                 _addr(d_total)), ctx)


def sharp_band_p2p_sharpen(ctx, windows, rank, w, h, row0, row1, epoch, params, out, grid_cap=0):
    arr = (_P * len(windows))(*windows)
    return _check(lib().sharp_band_p2p_sharpen(ctx, arr, len(windows), rank, w, h, row0, row1, int(epoch),
                                               _pp(params), _addr(out), int(grid_cap)), ctx)


def sharp_band_p2p_step(ctx, windows, rank, w, h, row0, row1, up_rows_own, epoch, params, out, grid_cap=0):
    arr = (_P * len(windows))(*windows)
    return _check(lib().sharp_band_p2p_step(ctx, arr, len(windows), rank, w, h, row0, row1, up_rows_own, int(epoch),
                                            _pp(params), _addr(out), int(grid_cap)), ctx)


def sharp_ipc_get_handle(d_ptr):
    """-> bytes (SHARP_IPC_HANDLE_BYTES) naming the allocation of d_ptr."""
    buf = ctypes.create_string_buffer(SHARP_IPC_HANDLE_BYTES)
    rc = lib().sharp_ipc_get_handle(d_ptr, buf)
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_ipc_get_handle: {sharp_strerror(rc)}")
    return buf.raw


def sharp_ipc_open_handle(handle):
    """-> device address (int) of a peer allocation mapped on this device."""
    buf = ctypes.create_string_buffer(bytes(handle), SHARP_IPC_HANDLE_BYTES)
    p = _P()
    rc = lib().sharp_ipc_open_handle(buf, ctypes.byref(p))
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_ipc_open_handle: {sharp_strerror(rc)}")
    return p.value


def sharp_ipc_close_handle(d_ptr):
    rc = lib().sharp_ipc_close_handle(d_ptr)
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_ipc_close_handle: {sharp_strerror(rc)}")


def sharp_set_path(ctx, path):
    return _check(lib().sharp_set_path(ctx, int(path)), ctx)


def sharp_get_path(ctx):
    return lib().sharp_get_path(ctx)


def sharp_get_stage_times(ctx):
    """-> dict stage name -> summed device ms (staged path, profiling on)."""
    arr = (ctypes.c_float * SHARP_NUM_STAGES)()
    _check(lib().sharp_get_stage_times(ctx, arr, SHARP_NUM_STAGES), ctx)
    return dict(zip(STAGE_NAMES, list(arr)))


def sharp_strerror(code):
    return lib().sharp_strerror(code).decode()


def sharp_last_error(ctx):
    return lib().sharp_last_error(ctx).decode()


def sharp_version():
    return lib().sharp_version().decode()


def sharp_band_halo(h, row0, row1):
    """-> (in0, in1): the image rows a band's input buffer must hold."""
    a, b = _I(), _I()
    rc = lib().sharp_band_halo(h, row0, row1, ctypes.byref(a), ctypes.byref(b))
    if rc != SHARP_OK:
        raise SharpError(rc, f"sharp_band_halo: {sharp_strerror(rc)}")
    return a.value, b.value


def sharp_band_edge_sum(ctx, band, w, h, row0, row1, d_partial):
    return _check(lib().sharp_band_edge_sum(ctx, _addr(band), w, h, row0, row1, _addr(d_partial)), ctx)


def sharp_band_sharpen(ctx, band, w, h, row0, row1, d_total, params, out):
    return _check(lib().sharp_band_sharpen(ctx, _addr(band), w, h, row0, row1, _addr(d_total), _pp(params),
                                           _addr(out)), ctx)


# ---------------------------------------------------------------- convenience
class Sharpener:
    """Owns one sharp_ctx.  Images: uint8 [H, W] (run) or [N, H, W] (run_batch)."""

    def __init__(self, device=-1, streams=0, chunk_frames=0, max_width=0, max_height=0, max_frames=0,
                 device_ids=None, shard=SHARP_SHARD_AUTO):
        """device_ids: a list of >= 2 device ordinals makes a multi-device
        context (sharp_config.num_devices / device_ids / shard)."""
        self.ctx = sharp_create(dict(device=device, streams=streams, chunk_frames=chunk_frames,
                                     max_width=max_width, max_height=max_height, max_frames=max_frames,
                                     device_ids=device_ids if device_ids and len(device_ids) > 1 else None,
                                     shard=shard))

    def close(self):
        if self.ctx:
            sharp_destroy(self.ctx)
            self.ctx = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @staticmethod
    def _shape(x):
        return tuple(x.shape)

    def _like(self, x):
        try:
            import torch
            if isinstance(x, torch.Tensor):
                return torch.empty_like(x)
        except ImportError:
            pass
        import numpy as np
        return np.empty_like(x)

    def set_stream(self, stream):
        sharp_set_stream(self.ctx, stream)

    def set_path(self, path):
        sharp_set_path(self.ctx, path)

    def stage_times(self):
        return sharp_get_stage_times(self.ctx)

    def run(self, img, params=None, out=None):
        H, W = self._shape(img)
        if out is None:
            out = self._like(img)
        sharp_run(self.ctx, img, W, H, params, out)
        return out

    def run_bands(self, bands, W, H, params=None, outs=None):
        """Device-resident row bands (one per device of the context)."""
        if outs is None:
            outs = [self._like(b) for b in bands]
        sharp_run_bands(self.ctx, bands, W, H, params, outs)
        return outs

    def run_batch(self, imgs, params=None, out=None):
        N, H, W = self._shape(imgs)
        if out is None:
            out = self._like(imgs)
        sharp_run_batch(self.ctx, imgs, N, W, H, params, out)
        return out

    def run_ex(self, imgs, params=None, out=None, flags=0, channels_last=False):
        """Any size >= 5, any strides (ROI views, interleaved channels with
        channels_last=True), in-place (out=imgs), reading switches `flags`."""
        n, c, h, w, li = layout_of(imgs, channels_last)
        if out is None:
            out = self._like(imgs)
        n2, c2, h2, w2, lo = layout_of(out, channels_last)
        if (n2, c2, h2, w2) != (n, c, h, w):
            raise ValueError("out must have the shape of imgs")
        sharp_run_ex(self.ctx, imgs, li, n, c, w, h, params, flags, out, lo)
        return out

    def enqueue_batch(self, d_imgs, d_outs, params=None):
        N, H, W = self._shape(d_imgs)
        sharp_enqueue_batch(self.ctx, d_imgs, N, W, H, params, d_outs)

    def stats(self):
        return sharp_get_stats(self.ctx)

    def batch_sums(self, n):
        return sharp_get_batch_sums(self.ctx, n)

    def set_profiling(self, enable=True):
        sharp_set_profiling(self.ctx, enable)

    def kernel_times(self):
        return sharp_get_kernel_times(self.ctx)

    # row bands of one image (orchestration in bands.py)
    def band_edge_sum(self, band, w, h, row0, row1, d_partial):
        sharp_band_edge_sum(self.ctx, band, w, h, row0, row1, d_partial)

    def band_sharpen(self, band, w, h, row0, row1, d_total, out, params=None):
        sharp_band_sharpen(self.ctx, band, w, h, row0, row1, d_total, params, out)
