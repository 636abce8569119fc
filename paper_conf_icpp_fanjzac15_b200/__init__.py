"""B200-native sharpness pipeline (Fan et al., ICPP 2015, sec. III).

Thin ctypes binding of the C ABI in include/sharp.h (libsharp.so, sm_100a).
Argument marshalling only: every step of the pipeline runs in the CUDA
kernels of libsharp.so.  There is NO CPU fallback -- if the library is
missing or no GPU is present, calls fail loudly.

Buffers may be torch tensors (CUDA or CPU, pinned or not), numpy arrays, or
raw integer addresses.  torch is used for device memory and streams only.
"""
from .binding import (  # noqa: F401
    SHARP_EINVAL,
    SHARP_ENOMEM,
    SHARP_ECUDA,
    SHARP_ENCCL,
    SHARP_ESTATE,
    SHARP_EUNSUPPORTED,
    SHARP_OK,
    LUT_SIZE,
    SharpError,
    SharpParams,
    SharpConfig,
    SharpStats,
    SharpKernelTimes,
    Sharpener,
    lib,
    library_path,
    sharp_create,
    sharp_default_params,
    sharp_destroy,
    sharp_enqueue_batch,
    sharp_get_batch_sums,
    sharp_get_stats,
    sharp_get_kernel_times,
    sharp_set_profiling,
    sharp_last_error,
    sharp_run,
    sharp_run_batch,
    sharp_set_stream,
    sharp_strerror,
    sharp_version,
    sharp_band_halo,
    sharp_band_edge_sum,
    sharp_band_sharpen,
    sharp_set_path,
    sharp_p2p_window_bytes,
    sharp_p2p_window_create,
    sharp_p2p_window_destroy,
    sharp_band_p2p_halo,
    sharp_band_p2p_allreduce,
    sharp_ipc_get_handle,
    sharp_ipc_open_handle,
    sharp_ipc_close_handle,
    SHARP_P2P_CTL_BYTES,
    sharp_get_path,
    sharp_get_stage_times,
    SHARP_PATH_AUTO,
    SHARP_PATH_STEP,
    SHARP_PATH_TWO_PASS,
    SHARP_PATH_STAGED,
    STAGE_NAMES,
)
