// Internal launch interface of the sm_100a kernels (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace sharp {

// Lookup tables built once per frame by the last CTA of pass 1: entry p
// (p = pEdge value, 0..1530 = 6*255) holds {adj(p), osc(p)} (R9, R11).
constexpr int kLutSize = 1536;
constexpr int kMaxRanks = 32;  // row bands of one image (peer-memory exchange slots)

struct Params {
  float amount, gamma, osc_gain, osc_scale;
  int flags = 0;  // reading switches, include/sharp.h SHARP_READ_*
};
// Reading switches (values of include/sharp.h SHARP_READ_*).
constexpr int kReadIntDownscale = 1;   // R2:  D = floor(block sum / 16)
constexpr int kReadColumnWins = 2;     // R5:  border column work after the row work
constexpr int kReadInteriorMean = 4;   // R8:  mean over the (W-2)(H-2) body
constexpr int kReadStrengthExp = 8;    // R9:  adj = A (1 - exp(-p / (K m)))
constexpr int kReadOscConst = 16;      // R11: oscStrength = G
constexpr int kReadTruncate = 32;      // R14: truncating output conversion
constexpr int kReadAll = 63;
// Switches that change per-pixel arithmetic (only the two-pass and staged
// paths implement them; the step kernel handles the LUT-only ones).
constexpr int kReadPerPixel = kReadIntDownscale | kReadColumnWins | kReadTruncate;

// Pass 1 (Sobel + reduction + LUT): for frames [0, n) of `imgs` (dense
// [n][H][W]) accumulates S into sums[frame_base + f] (must be zero on entry),
// and the last CTA of each frame writes means[frame_base + f] and
// luts[f * kLutSize ..] and re-arms counters[f] (must be zero on entry).
cudaError_t launch_edge_sum(const uint8_t *imgs, int n, int W, int H, const Params &p,
                            unsigned long long *sums, unsigned int *counters, float2 *luts,
                            double *means, cudaStream_t stream);

// Pass 2 (fused downscale/upscale/pError/Sobel/min-max/strength/preliminary/
// overshoot/output): frames [0, n) with the per-frame LUTs of pass 1.
cudaError_t launch_sharpen(const uint8_t *imgs, int n, int W, int H, const float2 *luts,
                           uint8_t *outs, int flags, cudaStream_t stream);

// General layouts (layout.cu): units u = f * C + c
// (frame f, channel c) of a strided source -> dense [units][H4][W4] with the
// last column / row replicated (R1'), and back (top-left w x h only).
// The padded units are [units][H4][P] (row pitch P >= W4; P = W4 is dense).
cudaError_t launch_gather(const uint8_t *src, size_t frame_stride, size_t pitch, int elem_stride, int C, int w,
                          int h, int W4, int H4, int P, int units, uint8_t *dst, cudaStream_t st);
cudaError_t launch_scatter(const uint8_t *src, int P, int H4, int units, int w, int h, uint8_t *dst,
                           size_t frame_stride, size_t pitch, int elem_stride, int C, cudaStream_t st);
cudaError_t preload_layout();

// TMA-staged, persistent, dynamically scheduled kernel (kernels_tma.cu) for a
// whole batch in ONE launch (pass 1, per-frame LUT build and pass 2 as tasks
// with in-kernel dependencies), used when tma_supported() (W % 16 == 0,
// W*H <= 2^29, 16-byte aligned input, 8-byte aligned output) or, for strided
// frames, tma_supported_strided().
struct BatchLaunch {
  const uint8_t *in = nullptr;  // [n][H][W]
  int n = 0;
  uint8_t *out = nullptr;       // [n][H][W]
  unsigned long long *acc = nullptr;   // n; zero on entry
  unsigned long long *sums = nullptr;  // n; out: S per frame
  double *means = nullptr;             // n; out: S / (W H)
  float2 *luts = nullptr;              // n * kLutSize (scratch)
  unsigned int *lut_done = nullptr;    // n; zero on entry
  unsigned int *lut_next = nullptr;    // n; zero on entry (res kernel: table chunks grabbed)
  unsigned int *task_counter = nullptr;  // 1; zero on entry
  // row-band launches only (launch_band_tma):
  unsigned long long *partial = nullptr;      // pass 1 out: the band's S
  const unsigned long long *total = nullptr;  // pass 2 in: the all-reduced S
  // strided frames (sharp_run_ex): bytes between rows / frames; 0 -> dense
  size_t in_pitch = 0, in_fs = 0, out_pitch = 0, out_fs = 0;
  // kStepBandFused: slot[rank] of every rank's window (peer mappings), this
  // rank's own slots, the epoch, the number of ranks; grid_cap > 0 limits the
  // persistent grid (several bands sharing one GPU must co-reside)
  unsigned long long *peer_slots[kMaxRanks] = {};
  const unsigned long long *my_slots = nullptr;
  unsigned long long epoch = 0;
  int ranks = 0, rank = 0, grid_cap = 0;
  // ... and the halo push in the same launch (halo_on): my window's control
  // words, the neighbours' (NULL at the image edges), where my first / last 4
  // rows go in their windows, and where they are in mine
  int halo_on = 0, halo_bytes = 0;
  unsigned long long *self_ctl = nullptr, *up_ctl = nullptr, *down_ctl = nullptr;
  uint8_t *up_halo = nullptr, *down_halo = nullptr;
  const uint8_t *own_top = nullptr, *own_bot = nullptr;
};
// Control words of a peer-memory window (bands_p2p.cu), u64 indices.
constexpr int kCtlDataUp = 64, kCtlDataDown = 65, kCtlReadyUp = 66, kCtlReadyDown = 67;
// Dense [n][H][W] frames: W % 16 == 0 (the TMA row stride), 16-byte aligned
// input, 8-byte aligned output, H >= 8, W * H <= 2^29.
bool tma_supported(const uint8_t *imgs, const uint8_t *outs, int W, int H);
// Strided frames: W % 8 == 0 (lane tiles end on the image's last column),
// in_pitch / in_fs multiples of 16 (TMA strides), out_pitch / out_fs
// multiples of 8 (8-byte stores), the same base alignments and limits.
bool tma_supported_strided(const uint8_t *imgs, size_t in_pitch, size_t in_fs, const uint8_t *outs, size_t out_pitch,
                           size_t out_fs, int W, int H);
cudaError_t launch_batch_tma(const BatchLaunch &a, int W, int H, const Params &p, cudaStream_t stream);

// TMEM-resident kernel (kernels_res.cu): pass 1 leaves each tile's pEdge in
// tensor memory, pass 2 of the same tile (same CTA) reads it back -- no
// second Sobel; the producers build a frame's tables while they wait for
// them.  Same frames / strides / scratch as launch_batch_tma plus lut_next.
// res_supported: frames of at most 2 x (resident grid) tiles of 960 x 12
// (~10 Mpx: up to 4K); else the step kernel.  Returns cudaErrorNotSupported
// when not applicable.
bool res_supported(int W, int H, int n);
cudaError_t launch_batch_res(const BatchLaunch &a, int W, int H, const Params &p, cudaStream_t stream);
cudaError_t preload_res();
// cuTensorMapEncodeTiled of [n][H][W] u8 frames at the given byte strides.
#include <cuda.h>
bool make_map(CUtensorMap *m, const uint8_t *imgs, int n, int W, int H, size_t pitch, size_t fs, int box_cols,
              int box_rows);

// One row band [row_lo, row_hi) of a W x H image (sec. 8(e)): a.in holds
// image rows [y0, y0 + rows_in) (the band plus its halo rows), a.out the
// band's rows (a.out = first output row).  mode kStepPass1 sums the band's
// pEdge into *a.partial (a.acc, a.task_counter zero on entry); kStepPass2
// builds the LUT from *a.total and writes the band (3 launches: arm, step,
// nothing else).  n = 1 frame; a.out is offset internally.
// kStepBandFused: pass 1, the cross-band all-reduce of S through peer
// memory (the partial slots of the bands_p2p.cu windows) and pass 2 of one
// band in ONE launch (a.peer_slots / a.my_slots / a.epoch / a.ranks).
enum StepMode { kStepAll = 0, kStepPass1 = 1, kStepPass2 = 2, kStepBandFused = 3 };
cudaError_t launch_band_tma(const BatchLaunch &a, int mode, int W, int H, int row_lo, int row_hi, int y0, int rows_in,
                            const Params &p, cudaStream_t stream);

// The paper's base design (kernels_staged.cu): one kernel per stage, every
// intermediate in HBM (the "base GPU" of sec. IV; first rung of the ladder).
enum Stage {
  kStageDownscale = 0, kStageBorder, kStageCenter, kStageSobel, kStageReduce, kStageStrength, kStageSharpen,
  kNumStages
};
// Optional per-stage event hook (profiling): begin(stage) / end(stage).
struct StageTimer {
  void *ctx = nullptr;
  void (*rec)(void *ctx, int stage, int begin, cudaStream_t st) = nullptr;
  void begin(int s, cudaStream_t st) const {
    if (rec) rec(ctx, s, 1, st);
  }
  void end(int s, cudaStream_t st) const {
    if (rec) rec(ctx, s, 0, st);
  }
};
size_t staged_scratch_bytes(int W, int H);
// One frame through K1..K7; *sum (u64) and *mean receive S and S / (W H).
cudaError_t launch_staged(const uint8_t *in, int W, int H, const Params &p, void *scratch,
                          unsigned long long *sum, double *mean, uint8_t *out, cudaStream_t st,
                          const StageTimer &timer);
constexpr int kStagedLaunches = 7;

// Scalar fused kernels (kernels_scalar.cu): one thread per pixel, stages fused
// (downscale, Sobel + reduction, table, everything else); table = false
// evaluates strength / oscStrength per pixel in f64 (the paper's fused
// kernel), true looks them up.  4 launches per frame.
size_t scalar_scratch_bytes(int W, int H);
cudaError_t launch_scalar(const uint8_t *in, int W, int H, const Params &p, void *scratch, unsigned long long *sum,
                          double *mean, uint8_t *out, bool table, cudaStream_t st);
cudaError_t preload_scalar();
constexpr int kScalarLaunches = 4;

// Fused peer-memory band exchange (bands_p2p.cu).
constexpr int kP2PCtlBytes = 1024;
constexpr int kP2PHalo = 4;
size_t p2p_window_bytes(int w, int rows_own);
cudaError_t launch_p2p_halo(uint8_t *self, int w, int rows_own, uint8_t *up, int up_rows_own, uint8_t *down,
                            unsigned long long epoch, cudaStream_t st);
cudaError_t launch_p2p_allreduce(uint8_t *const *windows, int G, int rank, const unsigned long long *partial,
                                 unsigned long long epoch, unsigned long long *total, cudaStream_t st);

// Under CUDA lazy module loading a kernel's module is loaded at its first
// launch, and that load can wait for the device to go idle -- a deadlock when
// an already running kernel spins on work the host has not launched yet (the
// peer-memory band exchange).  sharp_create loads every kernel up front.
cudaError_t preload_two_pass();
cudaError_t preload_staged();
cudaError_t preload_step();
cudaError_t preload_p2p();

// Kernel launches issued per (pass-1, pass-2) chunk.
constexpr int kLaunchesPerChunk = 2;

}  // namespace sharp
