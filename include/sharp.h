/*
 * include/sharp.h -- C ABI of the B200-native sharpness pipeline
 * (libsharp.so, built from paper_conf_icpp_fanjzac15_b200/csrc/).
 *
 * Method: M. Fan et al., "Optimizing Image Sharpening Algorithm on GPU",
 * ICPP 2015, section III: downscale (L130) -> upscale
 * border + body (L140-L146) -> pError (L148) -> Sobel pEdge (L158-L172) ->
 * global mean of pEdge (L174, the one global reduction) -> brightness
 * strength / adjusted pEdge (L178) -> preliminary sharpened image (L178) ->
 * overshoot control (L180-L212, Fig. 8) -> 8-bit image.  The readings of the
 * places where the paper is silent (R1..R16) are listed in DESIGN.md sec. 3;
 * the results are bit-identical to the CPU oracle in oracle/ (tests/).
 *
 * Conventions (all entry points):
 *  - Images are 8-bit single-channel, dense row-major, pitch == width
 *    ("4096 x 4096 bytes").  A batch is dense [n][h][w].
 *  - Width and height must be multiples of 4 and >= 8 (R1: the downscaled
 *    matrix is width/4 x height/4, L130); otherwise SHARP_EINVAL.
 *    (sharp_run_ex takes any size >= 5, strided / pitched / interleaved
 *    layouts, in-place calls and the reading switches.)
 *  - Pointers may be device pointers (on the context's device), pinned host
 *    or pageable host memory; the library classifies them
 *    (cudaPointerGetAttributes).  Host pointers go through pinned staging with
 *    H2D / compute / D2H overlapped across streams (sec. V-A).
 *  - Input and output must not overlap (in-place is rejected: the stencils
 *    read halos), else SHARP_EINVAL.  On any error `out` is left untouched
 *    unless the error is SHARP_ECUDA (device state unknown).
 *  - Ownership: the caller owns every image buffer; the library never retains
 *    them past return and never frees them.  The context owns all device
 *    scratch, streams, events and pinned staging; sharp_destroy releases them.
 *  - Synchrony: sharp_run / sharp_run_batch return after the output is
 *    complete.  sharp_enqueue_batch and the row-band calls are asynchronous
 *    on the context's stream (device pointers only).
 *  - Threads: a context is used by one thread at a time.
 *  - After a sticky CUDA error the context is poisoned: every later call
 *    returns SHARP_ESTATE until sharp_destroy.
 */
#ifndef SHARP_H
#define SHARP_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sharp_ctx sharp_ctx; /* opaque */

/* "User-defined parameters" of the strength (L178) and of the overshoot
 * tuning (L210).  Readings R9 / R11:
 *   adjusted pEdge  adj(p) = amount * (p / m)^gamma,  m = max(mean(pEdge), 1)
 *   oscStrength     osc(p) = clamp(osc_gain * exp(-p / (osc_scale * m)), 0, 1)
 * All must be finite and inside the ranges below, else SHARP_EINVAL. */
typedef struct {
  float amount;    /* A in [0, 16]       default 1.0 */
  float gamma;     /* gamma in [0, 4]    default 0.5 */
  float osc_gain;  /* G in [0, 1]        default 0.5 */
  float osc_scale; /* K in (0, 1e6]      default 2.0 */
} sharp_params;

typedef struct {
  int device;             /* CUDA device ordinal; -1 -> current device          */
  int max_width;          /* scratch pre-sizing hints; 0 -> grow on demand       */
  int max_height;
  int max_frames;
  int streams;            /* transfer pipeline depth for host buffers; 0 -> 3    */
  int chunk_frames;       /* frames per pass-1/pass-2 chunk; 0 -> automatic      */
  /* Several devices in ONE context.  num_devices
   * 0 or 1: the single device `device`.  num_devices G > 1: G devices
   * (device_ids[0..G-1], NULL -> 0..G-1; an ordinal may repeat, e.g. {0, 0}
   * to exercise the sharded paths on one GPU); the context keeps one
   * single-device context per entry and shards the work:
   *   SHARP_SHARD_FRAMES  sharp_run_batch splits the frames into G contiguous
   *                       ranges, one per device, run concurrently (frames
   *                       are independent: no data exchange);
   *   SHARP_SHARD_ROWS    sharp_run splits the image into G row bands (the
   *                       h/4 block rows split evenly, sharp_band_halo rows
   *                       of halo), sums the G partial pEdge sums (the L174
   *                       mean) and sharpens the bands -- bit-identical to
   *                       the single-device result;
   *   SHARP_SHARD_AUTO    frames for batches of >= 2 frames, rows for one image.
   * Multi-device contexts take HOST buffers in sharp_run / sharp_run_batch
   * (device-resident bands: sharp_run_bands); the other entry points return
   * SHARP_EUNSUPPORTED on them.  Ignored when num_devices <= 1. */
  int num_devices;
  const int *device_ids;  /* copied at sharp_create */
  int shard;              /* SHARP_SHARD_* */
} sharp_config;
enum { SHARP_SHARD_AUTO = 0, SHARP_SHARD_NONE = 1, SHARP_SHARD_ROWS = 2, SHARP_SHARD_FRAMES = 3 };

typedef struct {
  uint64_t edge_sum;  /* S = sum of pEdge over the image (frame 0 of a batch)    */
  double edge_mean;   /* S / (w*h)                                               */
  float device_ms;    /* device time of the last call (CUDA events)              */
  float total_ms;     /* host wall time of the last call                         */
  int frames;         /* frames processed by the last call                       */
  int kernels;        /* kernel launches issued by the last call                 */
} sharp_stats;

enum {
  SHARP_OK = 0,
  SHARP_EINVAL = -1,      /* bad argument (geometry, NULL, params, overlap)     */
  SHARP_ENOMEM = -2,      /* device or pinned allocation failed                 */
  SHARP_ECUDA = -3,       /* CUDA runtime / launch error                        */
  SHARP_ENCCL = -4,       /* multi-GPU communication error                      */
  SHARP_EUNSUPPORTED = -5,/* valid request this build cannot serve              */
  SHARP_ESTATE = -6       /* context poisoned by an earlier sticky error        */
};

/* Creates a context on cfg->device (NULL cfg -> defaults).  *ctx is set to
 * NULL on failure.  Returns SHARP_OK / SHARP_EINVAL / SHARP_ENOMEM / SHARP_ECUDA. */
int sharp_create(sharp_ctx **ctx, const sharp_config *cfg);

/* Releases everything the context owns.  NULL-safe. */
void sharp_destroy(sharp_ctx *ctx);

/* Fills *p with the defaults above (R16). */
void sharp_default_params(sharp_params *p);

/* Kernels are launched on `stream` (a cudaStream_t of the context's device,
 * e.g. torch.cuda.current_stream().cuda_stream); NULL restores the
 * context's own (non-blocking) stream -- pass cudaStreamLegacy ((void *)1)
 * for the legacy default stream. */
int sharp_set_stream(sharp_ctx *ctx, void *stream);

/* One image: img, out are w*h bytes.  params NULL -> defaults. */
int sharp_run(sharp_ctx *ctx, const uint8_t *img, int w, int h, const sharp_params *params,
              uint8_t *out);

/* n images, dense [n][h][w] in and out.  Frames are independent: each has its
 * own pEdge mean.  Host buffers are pipelined through pinned staging. */
int sharp_run_batch(sharp_ctx *ctx, const uint8_t *imgs, int n, int w, int h,
                    const sharp_params *params, uint8_t *outs);

/* Asynchronous variant for DEVICE pointers only: enqueues the whole batch on
 * the context's stream and returns (no host synchronisation; stats.device_ms
 * is not updated).  Used for graph capture / device-resident benchmarking. */
int sharp_enqueue_batch(sharp_ctx *ctx, const uint8_t *d_imgs, int n, int w, int h,
                        const sharp_params *params, uint8_t *d_outs);

/* ---- General geometry, layouts and reading switches (SURVEY.md sec. 8(f)
 * NEXT 3 and 4; DESIGN.md sec. 3 R1' and the R2/R5/R8/R9/R11/R14 switches).
 *
 * sharp_layout describes where the pixels of a batch live (all in bytes):
 * pixel (f, c, r, x) -- frame f, channel c, row r, column x -- is at
 *   base + f * frame_stride + c + r * pitch + x * elem_stride.
 * Zero fields take the dense defaults: elem_stride 1, pitch w * elem_stride,
 * frame_stride pitch * h.  A NULL layout is all defaults.  Requirements:
 * pitch >= w * elem_stride, frame_stride >= pitch * h, channels <= elem_stride.
 * So an ROI of a bigger image is {pitch = the big image's pitch}, an
 * interleaved C-channel image is {elem_stride = C} with channels = C, and a
 * planar one is C frames.
 *
 * sharp_run_ex sharpens the n * channels single-channel images ("units")
 * independently (each with its own pEdge mean: the method is
 * defined on one 8-bit matrix, so colour is handled per channel) and writes
 * them with out_layout.  Any w, h >= 5: when w or h is not a multiple of 4
 * (R1: the downscaled matrix is w/4 x h/4, L130) the unit is extended to the
 * next multiples of 4 by replicating its last column and last row, sharpened,
 * and cropped back (reading R1'; sharp_get_batch_sums then reports S of the
 * extended units).  In-place is allowed when imgs == outs with the same
 * layout; any other overlap is SHARP_EINVAL.  Pixels outside the w x h crops
 * (gaps between rows, other channels) are never modified.
 *
 * flags: reading switches, 0 = the default readings (bit-identical to
 * sharp_run_batch).  Each selects the alternative reading of a place where the
 * paper is silent; the CPU oracle implements the same switches.
 *   SHARP_READ_INT_DOWNSCALE  R2:  D = floor(block sum / 16) (the shift of L374)
 *   SHARP_READ_COLUMN_WINS    R5:  border column lines / copies after the row
 *                                  copies (top-left 2x2 from the column line)
 *   SHARP_READ_INTERIOR_MEAN  R8:  mean of pEdge over the (w-2)(h-2) body
 *   SHARP_READ_STRENGTH_EXP   R9:  adj(p) = amount * (1 - exp(-p / (osc_scale * m)))
 *   SHARP_READ_OSC_CONST      R11: oscStrength = osc_gain for every element
 *   SHARP_READ_TRUNCATE       R14: truncate instead of round-half-even
 * R8 / R9 / R11 only change the per-frame tables and run on every path; R2,
 * R5 and R14 change per-pixel arithmetic and run on the two-pass and staged
 * paths (SHARP_PATH_AUTO picks two-pass; SHARP_PATH_STEP returns
 * SHARP_EUNSUPPORTED).  Unknown bits -> SHARP_EINVAL.
 *
 * Dense single-channel inputs with w, h multiples of 4 take exactly the
 * sharp_run_batch path (host buffers pipelined, device buffers in one launch).
 * Single-channel DEVICE frames with w % 8 == 0 (w >= 16), h % 4 == 0, a 16-byte aligned
 * input with pitch / frame stride multiples of 16 and an 8-byte aligned output
 * with pitch / frame stride multiples of 8 (e.g. an aligned ROI) run straight
 * through the step kernel, zero-copy.  Everything else is gathered into padded
 * scratch on the device (host buffers: their byte range is copied up first),
 * run (on the step kernel when the padded width is a multiple of 8), and
 * scattered back, one chunk of frames at a time.  Synchronous. */
typedef struct {
  size_t pitch;        /* bytes from one row to the next          (0 -> w * elem_stride) */
  size_t frame_stride; /* bytes from one frame to the next        (0 -> pitch * h)       */
  int elem_stride;     /* bytes from one pixel to the next in a row (0 -> 1)             */
} sharp_layout;
enum {
  SHARP_READ_INT_DOWNSCALE = 1,
  SHARP_READ_COLUMN_WINS = 2,
  SHARP_READ_INTERIOR_MEAN = 4,
  SHARP_READ_STRENGTH_EXP = 8,
  SHARP_READ_OSC_CONST = 16,
  SHARP_READ_TRUNCATE = 32
};
int sharp_run_ex(sharp_ctx *ctx, const uint8_t *imgs, const sharp_layout *in_layout, int n, int channels, int w,
                 int h, const sharp_params *params, int flags, uint8_t *outs, const sharp_layout *out_layout);

/* Statistics of the last completed call. */
int sharp_get_stats(const sharp_ctx *ctx, sharp_stats *s);

/* Per-frame pEdge sums S of the last run / enqueued batch (waits for the
 * context's stream).  n must not exceed the number of frames of that call. */
int sharp_get_batch_sums(sharp_ctx *ctx, uint64_t *sums, int n);

/* ---- Row-band sharding of ONE image.
 * The image is split into row bands, one per process / GPU.  The only
 * coupling between bands is the global pEdge mean ("the
 * arithmetic mean of the elements in this matrix"), so a band runs in two
 * calls around one all-reduce of a 64-bit sum:
 *   1. sharp_band_edge_sum  -> *d_partial = sum of pEdge over rows [row0, row1)
 *   2. the caller sums the partials of all bands into *d_total (e.g. NCCL
 *      all-reduce through torch.distributed)
 *   3. sharp_band_sharpen   -> output rows [row0, row1), bit-identical to the
 *      same rows of sharp_run on the whole image.
 * Geometry: band g owns output rows [row0, row1), multiples of 4 with
 * 0 <= row0 < row1 <= h, so no 4x4 downscale block straddles two bands.  Its
 * input `band` holds image rows [in0, in1) = [max(row0-4, 0), min(row1+4, h))
 * (sharp_band_halo): the band plus 4 halo rows on each side -- the upscale of
 * rows row0 .. row1-1 reads D rows row0/4-1 .. row1/4 (L146), the Sobel and
 * the 3x3 overshoot window one row (L158-L172, L182).  Rows are dense, pitch w.
 * Requirements: DEVICE pointers on the context's device; w % 16 == 0, `band`
 * 16-byte aligned, `out` 8-byte aligned (the TMA path), w*h < 2^29 -- else
 * SHARP_EUNSUPPORTED / SHARP_EINVAL.  d_partial / d_total: device uint64.
 * Both calls are asynchronous on the context's stream (sharp_set_stream);
 * `out` ((row1-row0) x w bytes) must not overlap `band`. */
int sharp_band_halo(int h, int row0, int row1, int *in0, int *in1);
int sharp_band_edge_sum(sharp_ctx *ctx, const uint8_t *band, int w, int h, int row0, int row1,
                        uint64_t *d_partial);
int sharp_band_sharpen(sharp_ctx *ctx, const uint8_t *band, int w, int h, int row0, int row1,
                       const uint64_t *d_total, const sharp_params *params, uint8_t *out);

/* ---- Device-resident row bands over the devices of a multi-device context
 * (SURVEY.md sec. 8(b) / 8(e) 2).  bands[g] / outs[g]: DEVICE pointers on
 * device_ids[g] holding rows [row0_g, row1_g) of the w x h image (dense, pitch
 * w), the partition of sharp_band_rows (the h/4 block rows split as evenly as
 * possible, the first (h/4) % G bands one block row longer).  The library
 * copies each band with its 4-row halos (the neighbours' edge rows, peer
 * copies) into its own scratch, sums the bands' partial pEdge sums (L174:
 * one global mean) and writes outs[g] = rows [row0_g, row1_g) of the result,
 * bit-identical to sharp_run on the whole image.  Synchronous.  A
 * single-device context takes G = 1 (bands[0] = the whole image).
 * Requirements as for sharp_band_edge_sum (w % 16 == 0, w * h < 2^29). */
int sharp_band_rows(int h, int n_bands, int band, int *row0, int *row1);
int sharp_run_bands(sharp_ctx *ctx, const uint8_t *const *bands, int w, int h, const sharp_params *params,
                    uint8_t *const *outs);

/* ---- Fused peer-memory band exchange (
 * DESIGN.md sec. 9): the same two couplings as above -- 4 halo rows per side
 * and the 64-bit pEdge sum -- moved by direct stores into the neighbours' /
 * every rank's memory (NVLink peer mappings from CUDA IPC) with epoch flags,
 * instead of NCCL: one single-CTA kernel per exchange, no host round trip.
 *
 * Each rank owns a zero-initialised device "window" of
 * sharp_p2p_window_bytes(w, rows_own) bytes (16-byte aligned):
 *   [0, SHARP_P2P_CTL_BYTES)  control words (flags, partial slots; library-owned)
 *   then rows of pitch w: 4 halo rows | the band's rows_own own rows | 4 halo rows.
 * The caller writes its own rows at offset SHARP_P2P_CTL_BYTES + 4*w; after
 * sharp_band_p2p_halo the window rows [in0 - (row0 - 4), ...) are exactly the
 * band input of sharp_band_edge_sum / sharp_band_sharpen (for the first band
 * skip the upper halo rows, for the last the lower ones).
 * sharp_band_p2p_halo: pushes this band's first/last 4 own rows into the
 *   neighbours' halos (up_window / down_window: their windows as mapped on
 *   this device, NULL at the image edges; up_rows_own: the upper band's own
 *   rows), publishes them with `epoch`, and returns (asynchronously) when
 *   both neighbours' rows for `epoch` have arrived in ours.
 * sharp_band_p2p_allreduce: stores (epoch, *d_partial) into slot `rank` of
 *   every window (windows: HOST array of the n_ranks windows as mapped on this
 *   device, windows[rank] = ours), waits for all n_ranks slots of ours and
 *   writes their sum to *d_total (device u64).
 * Every rank must make the same sequence of calls with epochs 1, 2, 3, ...
 * (one per image); w % 16 == 0, rows_own >= 4, n_ranks <= 32; both calls are
 * asynchronous on the context's stream and wait on the device for the peers.
 * sharp_ipc_*: thin wrappers of cudaIpcGetMemHandle / cudaIpcOpenMemHandle
 * (lazy peer access) / cudaIpcCloseMemHandle for exchanging the windows
 * between processes (handles are SHARP_IPC_HANDLE_BYTES opaque bytes). */
#define SHARP_P2P_CTL_BYTES 1024
#define SHARP_IPC_HANDLE_BYTES 64
size_t sharp_p2p_window_bytes(int w, int rows_own); /* 0 on bad arguments */
/* cudaMalloc + zero of one window on the current device (its own allocation,
 * so an IPC handle of it maps exactly the window); the caller owns it and
 * releases it with sharp_p2p_window_destroy (after closing peer mappings). */
int sharp_p2p_window_create(int w, int rows_own, void **d_window);
void sharp_p2p_window_destroy(void *d_window);
int sharp_band_p2p_halo(sharp_ctx *ctx, uint8_t *self_window, int w, int rows_own, uint8_t *up_window,
                        int up_rows_own, uint8_t *down_window, uint64_t epoch);
int sharp_band_p2p_allreduce(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank,
                             const uint64_t *d_partial, uint64_t epoch, uint64_t *d_total);
/* sharp_band_p2p_sharpen: pass 1, the cross-band all-reduce of the pEdge
 * partials and pass 2 of this band in ONE persistent launch -- the step
 * kernel's LUT tasks publish the band's partial into slot `rank` of every
 * window (the same epoch-parity slots as sharp_band_p2p_allreduce) and poll
 * this window's n_ranks slots for `epoch`, so the collective runs inside the
 * compute kernel over NVLink.  Call after sharp_band_p2p_halo of the same
 * epoch (the band's input is its window's rows); writes rows [row0, row1)
 * to `out` (device, 8-byte aligned, (row1-row0) x w).  grid_cap > 0 limits
 * the persistent grid (CTAs): bands that share ONE GPU must co-reside, so
 * their caps must sum to at most 3 x SMs (one band per GPU: 0 = all SMs).
 * Asynchronous on the context's stream. */
int sharp_band_p2p_sharpen(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank, int w, int h, int row0,
                           int row1, uint64_t epoch, const sharp_params *params, uint8_t *out, int grid_cap);
/* sharp_band_p2p_step: the same launch with the halo push folded in -- the
 * kernel's first task sets this band's "ready" flags in the neighbours'
 * windows, waits for theirs, and its warps store the band's first / last 4
 * rows into the neighbours' halos with a system-wide fence and "data" flags;
 * the pass-1 tiles at the band's edges wait for the neighbours' data flags.
 * ONE launch per band per image (no sharp_band_p2p_halo call).  up_rows_own:
 * the upper band's own row count (for its lower halo).  All bands of an image
 * must run it concurrently (on one GPU: grid caps summing to at most 3 x SMs). */
int sharp_band_p2p_step(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank, int w, int h, int row0,
                        int row1, int up_rows_own, uint64_t epoch, const sharp_params *params, uint8_t *out,
                        int grid_cap);
int sharp_ipc_get_handle(const void *d_ptr, void *handle);
int sharp_ipc_open_handle(const void *handle, void **d_ptr);
int sharp_ipc_close_handle(void *d_ptr);

/* Per-kernel device time accounting (CUDA events around every launch, on
 * the launch stream).  enable != 0 starts (and resets) accounting. */
typedef struct {
  float pass1_ms;      /* generic path: summed duration of edge_sum launches        */
  float pass2_ms;      /* generic path: summed duration of sharpen launches         */
  int pass1_launches;
  int pass2_launches;
  float step_ms;       /* TMA path: summed duration of step launches (pass 1 of
                          chunk c+1 fused with pass 2 of chunk c)                  */
  int step_launches;
  double pixels;       /* output pixels completed by the accounted launches         */
} sharp_kernel_times;
int sharp_set_profiling(sharp_ctx *ctx, int enable);
/* Waits for the launch stream, then returns the accumulated times. */
int sharp_get_kernel_times(sharp_ctx *ctx, sharp_kernel_times *t);

/* ---- Kernel paths: the optimisation ladder of PAPER.md sec. V (Fig. 12,
 * Fig. 14), every rung bit-identical to the oracle.
 *   SHARP_PATH_AUTO     the TMA kernels where they apply -- the resident kernel for launches of
 *                       1 to 100 Mpx, the step kernel otherwise (measured crossovers) -- else the
 *                       two-pass path (default)
 *   SHARP_PATH_STEP     one persistent TMA-staged launch per batch (kernels_tma.cu): pass 1,
 *                       per-frame LUT and pass 2 as dynamically scheduled tasks with
 *                       in-kernel dependencies; needs w % 16 == 0 (sharp_run_ex: any w % 8 == 0,
 *                       w >= 16, through strided tensor maps), 16-byte aligned input,
 *                       8-byte aligned output, w*h <= 2^29, else SHARP_EUNSUPPORTED
 *   SHARP_PATH_RES      one persistent TMA-staged launch per batch whose pass 1 leaves each
 *                       tile's pEdge in tensor memory for pass 2 of the same tile (kernels_res.cu:
 *                       no second Sobel, no pEdge traffic); the step kernel's geometry rules plus
 *                       at most 2 x (resident grid) tiles of 960 x 12 per frame (up to ~10 Mpx,
 *                       4K included), else SHARP_EUNSUPPORTED
 *   SHARP_PATH_TWO_PASS two fused kernels per chunk of frames (kernels.cu): Sobel +
 *                       reduction + LUT, then everything else; any w % 4 == 0
 *   SHARP_PATH_FUSED    scalar fused kernels (kernels_scalar.cu): one thread per pixel, no SIMD
 *                       or data reuse, the stages fused into downscale / Sobel + reduction /
 *                       table / everything else (4 launches per frame; sec. V-B "kernel fusion")
 *   SHARP_PATH_FUSED_EXP the same with strength and oscStrength evaluated per pixel in f64 (the
 *                       "many exponentiations" of L232) instead of the per-frame table
 *   SHARP_PATH_STAGED   the paper's BASE GPU design (sec. IV): one kernel per
 *                       stage, every intermediate matrix in HBM (kernels_staged.cu,
 *                       7 launches per frame); the per-stage breakdown of Fig. 13
 * Takes effect at the next call.  Row-band calls need AUTO or STEP.  Environment
 * SHARP_FORCE_GENERIC=1 at sharp_create selects SHARP_PATH_TWO_PASS. */
enum {
  SHARP_PATH_AUTO = 0,
  SHARP_PATH_STEP = 1,
  SHARP_PATH_TWO_PASS = 2,
  SHARP_PATH_STAGED = 3,
  SHARP_PATH_RES = 4,
  SHARP_PATH_FUSED = 5,
  SHARP_PATH_FUSED_EXP = 6
};
int sharp_set_path(sharp_ctx *ctx, int path);
int sharp_get_path(const sharp_ctx *ctx);

/* Staged path + profiling: device ms per stage (CUDA events around each
 * launch, summed since sharp_set_profiling(ctx, 1)); ms[SHARP_NUM_STAGES]
 * in the order below (sec. III / Fig. 13).  Waits for the events. */
enum {
  SHARP_STAGE_DOWNSCALE = 0, /* K1  O -> D (L130)                         */
  SHARP_STAGE_BORDER,        /* K2  D -> U ring, steps i-vii (L140-L142)  */
  SHARP_STAGE_CENTER,        /* K3  D -> U body (L146)                    */
  SHARP_STAGE_SOBEL,         /* K4  O -> pEdge (L158-L172)                */
  SHARP_STAGE_REDUCE,        /* K5  pEdge -> S (L174)                     */
  SHARP_STAGE_STRENGTH,      /* K6  pEdge, S -> adj, osc per pixel (L178) */
  SHARP_STAGE_SHARPEN,       /* K7  O, U, adj, osc -> out (L178-L212)     */
  SHARP_NUM_STAGES
};
int sharp_get_stage_times(sharp_ctx *ctx, float *ms, int n);

/* Static strings. */
const char *sharp_strerror(int code);
const char *sharp_last_error(const sharp_ctx *ctx);

/* Library build / kernel information (e.g. "sm_100a ..."). */
const char *sharp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SHARP_H */
