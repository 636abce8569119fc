// C ABI + runtime of libsharp.so (include/sharp.h).
//
// The runtime owns: the device scratch of the two passes (per-frame u64 edge
// sums, per-frame means, per-chunk-frame counters and lookup tables), the
// stream it launches on, a pipeline of `streams` slots (stream + device
// in/out buffers + pinned host staging) used when the caller passes host
// memory (sec. V-A: bulk read/write transfers, only O up and the
// final image down, L252-L266, L336), and the error state.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <thread>
#include <vector>

#include "kernels.h"
#include "sharp.h"

namespace {

// Host copies between pageable user memory and the pinned staging: split over
// up to 8 threads (one thread moves ~10 GB/s; the pipeline's PCIe leg ~50).
void par_memcpy(void *dst, const void *src, size_t n) {
  const size_t kMinPart = 4u << 20;
  const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
  const size_t parts = std::min<size_t>(std::min(8u, hw), std::max<size_t>(1, n / kMinPart));
  if (parts <= 1) {
    memcpy(dst, src, n);
    return;
  }
  std::vector<std::thread> th;
  const size_t step = (n + parts - 1) / parts;
  for (size_t i = 1; i < parts; ++i) {
    const size_t a = i * step, b = std::min(n, a + step);
    if (a < b) th.emplace_back([=] { memcpy((char *)dst + a, (const char *)src + a, b - a); });
  }
  memcpy(dst, src, std::min(n, step));
  for (auto &t : th) t.join();
}

constexpr size_t kL2ChunkBudget = 24u << 20;  // input bytes per chunk kept L2-resident between passes
// Host pipeline on the step kernel (no L2 residency needed between launches):
// bigger chunks amortise the per-chunk copy / launch overheads (measured on
// 1024 x 1080p pinned: 24 MB chunks 47.4 ms, 48-64 MB 45.3-46.3 ms, PCIe
// ceiling with both directions busy 43.3 ms; tools/e2e_sweep.py).
constexpr size_t kHostStepChunkBudget = 48u << 20;
constexpr int kMaxSlots = 8;
// SHARP_PATH_AUTO's choice of the TMEM-resident kernel (launch pixels), from
// tools/step_time.py sweeps on B200 (device-resident, back-to-back calls):
// it wins from ~1 Mpx (below, its one 16-warp CTA per SM costs more than it
// saves; 512^2: 18.5 vs 17.5 us) up to ~16 Mpx per launch (1080p x1 18.8 vs
// 20.9 us, x2 20.5 vs 21.9, 4K x1 28.7 vs 29.7, 720p x16 49.5 vs 57.0); from
// there the step kernel with compact / lagged schedules is as fast or faster
// (1080p x8 41.2 vs 43.1 us, 4K x2 41.1 vs 44.2, x4 64.0 vs 75.8, x8 111 vs
// 128; 1080p x16..48 within 1%).
constexpr double kResAutoMinPx = 1.0e6, kResAutoMaxPx = 1.6e7;

struct Slot {
  cudaStream_t stream = nullptr;
  cudaEvent_t done = nullptr;
  uint8_t *d_in = nullptr, *d_out = nullptr;   // device staging (chunk)
  uint8_t *h_in = nullptr, *h_out = nullptr;   // pinned staging (chunk)
  unsigned int *counters = nullptr;            // per chunk frame
  float2 *luts = nullptr;                      // per chunk frame
  // SHARP_PATH_STAGED scratch (D, U, pEdge, strength of one frame): one per
  // slot, since the host pipeline runs the slots' chunks concurrently
  void *staged = nullptr;
  size_t staged_cap = 0;
};

}  // namespace

struct sharp_ctx {
  int device = 0;
  cudaStream_t own_stream = nullptr;
  cudaStream_t stream = nullptr;  // launch stream (own or caller's)
  cudaEvent_t ev_start = nullptr, ev_stop = nullptr;
  struct HostStats { unsigned long long sum; double mean; } *h_stats = nullptr;  // pinned
  int nslots = 3;
  int chunk_cfg = 0;
  int path = SHARP_PATH_AUTO;  // SHARP_FORCE_GENERIC=1 at sharp_create selects SHARP_PATH_TWO_PASS
  cudaEvent_t stage_open[sharp::kNumStages] = {};
  Slot slots[kMaxSlots];
  size_t slot_chunk_frames = 0, slot_stage_bytes = 0;  // capacity of the slot buffers
  void *zero_block = nullptr;  // acc | sums | lut_done | tcounters (one memset per call)
  size_t zero_bytes = 0;
  unsigned long long *sums = nullptr;
  double *means = nullptr;
  size_t frames_cap = 0;
  unsigned int *tcounters = nullptr;  // dynamic-scheduling task counters, one per step launch
  size_t tcounters_cap = 0;
  unsigned int *lut_done = nullptr;   // per frame: finished LUT-task warps / table chunks
  unsigned int *lut_next = nullptr;   // per frame: table chunks grabbed (resident kernel)
  unsigned long long *acc = nullptr;  // per frame: pass-1 arrivals << 40 | partial sum (batch kernel)
  float2 *luts = nullptr;             // per frame lookup tables (batch kernel)
  // general layouts (sharp_run_ex): dense padded in / out, device copies of host byte ranges
  uint8_t *gx_in = nullptr, *gx_out = nullptr, *gx_src = nullptr, *gx_dst = nullptr;
  size_t gx_cap = 0, gx_out_cap = 0, gx_src_cap = 0, gx_dst_cap = 0;
  int last_frames = 0;
  sharp_stats stats{};
  // profiling: event pairs around launches (kind 1 = pass 1, 2 = pass 2,
  // 3 = step kernel, 10 + s = stage s of the staged path)
  bool profiling = false;
  struct Rec { cudaEvent_t a, b; int kind; double px; };
  std::vector<Rec> recs;
  std::vector<cudaEvent_t> ev_pool;
  bool poisoned = false;
  char err[256] = {0};
  // Multi-device context (sharp_config.num_devices > 1): one single-device
  // context per entry of device_ids; this one owns no device resources but
  // the per-band scratch below (allocated on the sub-contexts' devices).
  std::vector<sharp_ctx *> sub;
  int shard = SHARP_SHARD_AUTO;
  std::vector<std::pair<int, int>> last_split;  // frame ranges of the last sharded batch
  struct BandBuf {
    uint8_t *in = nullptr, *out = nullptr;
    size_t in_cap = 0, out_cap = 0;
    unsigned long long *part = nullptr, *total = nullptr;  // device u64
    unsigned long long *h = nullptr;                       // pinned: [0] partial, [1] total
  };
  std::vector<BandBuf> bb;
};

namespace {

int set_err(sharp_ctx *c, int code, const char *fmt, const char *what) {
  if (c) snprintf(c->err, sizeof(c->err), fmt, what);
  return code;
}

// Maps a CUDA error to a return code; sticky errors poison the context.
int cuda_fail(sharp_ctx *c, cudaError_t e, const char *where) {
  if (e == cudaSuccess) return SHARP_OK;
  if (c) {
    snprintf(c->err, sizeof(c->err), "%s: %s", where, cudaGetErrorString(e));
    if (e == cudaErrorMemoryAllocation) {
      cudaGetLastError();
      return SHARP_ENOMEM;
    }
    // Probe whether the error is sticky (the context is unusable).
    cudaError_t probe = cudaDeviceSynchronize();
    if (probe != cudaSuccess) c->poisoned = true;
    cudaGetLastError();
  }
  return SHARP_ECUDA;
}

#define CK(expr)                                          \
  do {                                                    \
    cudaError_t e__ = (expr);                             \
    if (e__ != cudaSuccess) return cuda_fail(ctx, e__, #expr); \
  } while (0)

// Paths served by the TMA-staged kernels (the resident kernel or the step kernel).
bool tma_family(int path) { return path == SHARP_PATH_AUTO || path == SHARP_PATH_STEP || path == SHARP_PATH_RES; }

bool params_ok(const sharp_params &p) {
  // R16 ranges; NaN fails every comparison.
  return p.amount >= 0.0f && p.amount <= 16.0f && p.gamma >= 0.0f && p.gamma <= 4.0f &&
         p.osc_gain >= 0.0f && p.osc_gain <= 1.0f && p.osc_scale > 0.0f && p.osc_scale <= 1.0e6f;
}

enum Kind { kDevice, kPinned, kPageable };

int classify(sharp_ctx *ctx, const void *p, Kind *k) {
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *k = kPageable;
    return SHARP_OK;
  }
  switch (a.type) {
    case cudaMemoryTypeDevice:
    case cudaMemoryTypeManaged:
      if (a.device != ctx->device)
        return set_err(ctx, SHARP_EINVAL, "%s", "device pointer belongs to another device");
      *k = kDevice;
      break;
    case cudaMemoryTypeHost: *k = kPinned; break;
    default: *k = kPageable;
  }
  return SHARP_OK;
}

// Per-frame scratch.  acc, sums, lut_done and the task counters live in ONE
// allocation ("zero block") so a call zeroes them with a single memset (for a
// single image the memsets are a visible share of the latency).
int ensure_frames(sharp_ctx *ctx, size_t n, size_t n_tc = 0) {
  const size_t need_tc = std::max(n_tc, 2 * n + 2);
  if (n <= ctx->frames_cap && need_tc <= ctx->tcounters_cap) return SHARP_OK;
  CK(cudaStreamSynchronize(ctx->stream));
  for (int i = 0; i < ctx->nslots; ++i) CK(cudaStreamSynchronize(ctx->slots[i].stream));
  cudaFree(ctx->zero_block);
  cudaFree(ctx->means);
  cudaFree(ctx->luts);
  ctx->zero_block = nullptr;
  ctx->sums = ctx->acc = nullptr;
  ctx->lut_done = ctx->lut_next = ctx->tcounters = nullptr;
  ctx->means = nullptr;
  ctx->luts = nullptr;
  ctx->frames_cap = ctx->tcounters_cap = ctx->zero_bytes = 0;
  const size_t cap = std::max(n, ctx->frames_cap), tcap = std::max(need_tc, 2 * cap + 2);
  const size_t b_acc = cap * 8, b_sums = cap * 8, b_done = (cap * 4 + 7) & ~(size_t)7, b_tc = tcap * 4;
  CK(cudaMalloc(&ctx->zero_block, b_acc + b_sums + 2 * b_done + b_tc));
  uint8_t *z = static_cast<uint8_t *>(ctx->zero_block);
  ctx->acc = reinterpret_cast<unsigned long long *>(z);
  ctx->sums = reinterpret_cast<unsigned long long *>(z + b_acc);
  ctx->lut_done = reinterpret_cast<unsigned int *>(z + b_acc + b_sums);
  ctx->lut_next = reinterpret_cast<unsigned int *>(z + b_acc + b_sums + b_done);
  ctx->tcounters = reinterpret_cast<unsigned int *>(z + b_acc + b_sums + 2 * b_done);
  ctx->zero_bytes = b_acc + b_sums + 2 * b_done + b_tc;
  CK(cudaMalloc(&ctx->means, cap * sizeof(double)));
  CK(cudaMalloc(&ctx->luts, cap * sharp::kLutSize * sizeof(float2)));
  ctx->frames_cap = cap;
  ctx->tcounters_cap = tcap;
  return SHARP_OK;
}

int ensure_task_counters(sharp_ctx *ctx, size_t n) { return ensure_frames(ctx, ctx->frames_cap, n); }

void free_slot(Slot &s) {
  cudaFree(s.d_in);
  cudaFree(s.d_out);
  cudaFreeHost(s.h_in);
  cudaFreeHost(s.h_out);
  cudaFree(s.counters);
  cudaFree(s.luts);
  cudaFree(s.staged);
  s.staged = nullptr;
  s.staged_cap = 0;
  s.d_in = s.d_out = s.h_in = s.h_out = nullptr;
  s.counters = nullptr;
  s.luts = nullptr;
}

// Every slot gets counters + LUTs for `chunk` frames; device/pinned staging
// buffers of chunk*frame_bytes only when `staging` (host-memory calls).
int ensure_slots(sharp_ctx *ctx, size_t chunk, size_t frame_bytes, bool staging) {
  const size_t need_stage = staging ? chunk * frame_bytes : 0;
  if (chunk <= ctx->slot_chunk_frames && need_stage <= ctx->slot_stage_bytes) return SHARP_OK;
  CK(cudaStreamSynchronize(ctx->stream));
  for (int i = 0; i < ctx->nslots; ++i) CK(cudaStreamSynchronize(ctx->slots[i].stream));
  const size_t cap = std::max(chunk, ctx->slot_chunk_frames);
  const size_t stage = std::max(need_stage, ctx->slot_stage_bytes);
  ctx->slot_chunk_frames = 0;
  ctx->slot_stage_bytes = 0;
  for (int i = 0; i < ctx->nslots; ++i) {
    Slot &s = ctx->slots[i];
    free_slot(s);
    CK(cudaMalloc(&s.counters, cap * sizeof(unsigned int)));
    CK(cudaMemset(s.counters, 0, cap * sizeof(unsigned int)));
    CK(cudaMalloc(&s.luts, 2 * cap * sharp::kLutSize * sizeof(float2)));  // two chunk parities
    if (stage) {
      CK(cudaMalloc(&s.d_in, stage));
      CK(cudaMalloc(&s.d_out, stage));
      CK(cudaHostAlloc(&s.h_in, stage, cudaHostAllocDefault));
      CK(cudaHostAlloc(&s.h_out, stage, cudaHostAllocDefault));
    }
  }
  ctx->slot_chunk_frames = cap;
  ctx->slot_stage_bytes = stage;
  return SHARP_OK;
}

size_t chunk_frames(const sharp_ctx *ctx, size_t frame_bytes, int n, size_t budget = kL2ChunkBudget) {
  size_t c = ctx->chunk_cfg > 0 ? (size_t)ctx->chunk_cfg : std::max<size_t>(1, budget / frame_bytes);
  c = std::min<size_t>(c, 65535);
  return std::min<size_t>(c, (size_t)n);
}

int validate(sharp_ctx *ctx, const void *in, const void *out, int n, int w, int h, const sharp_params *p) {
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  if (!in || !out) return set_err(ctx, SHARP_EINVAL, "%s", "NULL image pointer");
  if (n < 1) return set_err(ctx, SHARP_EINVAL, "%s", "n < 1");
  if (w < 8 || h < 8 || (w & 3) || (h & 3))
    return set_err(ctx, SHARP_EINVAL, "%s", "width and height must be multiples of 4 and >= 8 (R1)");
  if ((long long)w * h >= (1ll << 31) || w > 65536 || h > 65536)
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "image larger than 2^31 pixels");
  if (p && !params_ok(*p)) return set_err(ctx, SHARP_EINVAL, "%s", "parameter out of range or not finite");
  const size_t bytes = (size_t)n * w * h;
  const uintptr_t a = (uintptr_t)in, b = (uintptr_t)out;
  if (a < b + bytes && b < a + bytes) return set_err(ctx, SHARP_EINVAL, "%s", "input and output overlap");
  return SHARP_OK;
}

cudaEvent_t pool_event(sharp_ctx *ctx) {
  if (!ctx->ev_pool.empty()) {
    cudaEvent_t e = ctx->ev_pool.back();
    ctx->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  if (cudaEventCreate(&e) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return e;
}

// Records an event pair around `launch` when profiling.
template <typename F>
cudaError_t timed(sharp_ctx *ctx, cudaStream_t st, int kind, double px, F launch) {
  if (!ctx->profiling) return launch();
  cudaEvent_t a = pool_event(ctx), b = pool_event(ctx);
  if (!a || !b) return launch();
  cudaEventRecord(a, st);
  cudaError_t e = launch();
  cudaEventRecord(b, st);
  ctx->recs.push_back({a, b, kind, px});
  return e;
}

// Staged-path scratch of a slot for one w x h frame (grown on demand).
int rc_staged(sharp_ctx *ctx, Slot &slot, cudaStream_t st, int w, int h) {
  const size_t need = std::max(sharp::staged_scratch_bytes(w, h), sharp::scalar_scratch_bytes(w, h));
  if (need <= slot.staged_cap) return SHARP_OK;
  cudaStreamSynchronize(st);
  cudaStreamSynchronize(ctx->stream);
  cudaFree(slot.staged);
  slot.staged = nullptr;
  slot.staged_cap = 0;
  if (cudaMalloc(&slot.staged, need) != cudaSuccess) {
    cudaGetLastError();
    return SHARP_ENOMEM;
  }
  slot.staged_cap = need;
  return SHARP_OK;
}

// StageTimer hook: an event pair per stage launch (profiling only).
void stage_rec(void *vctx, int stage, int begin, cudaStream_t st) {
  sharp_ctx *ctx = static_cast<sharp_ctx *>(vctx);
  cudaEvent_t e = pool_event(ctx);
  if (!e) return;
  cudaEventRecord(e, st);
  if (begin) {
    ctx->stage_open[stage] = e;
  } else if (ctx->stage_open[stage]) {
    ctx->recs.push_back({ctx->stage_open[stage], e, 10 + stage, 0.0});
    ctx->stage_open[stage] = nullptr;
  }
}

// Device-resident batch on one stream, in chunks of frames.
//  * TMA path: launch c = pass 1 of chunk c + pass 2 of chunk c-1 (one
//    dynamically scheduled step kernel); chunk c's input is still in L2 when
//    launch c+1 re-reads it.  LUT buffers alternate between chunk parities.
//  * generic path: pass 1 then pass 2 per chunk.
// `tc` points at this call's zeroed task counters (one per step launch).
// Byte strides of device frames (0 = dense); only the step kernel takes
// strided frames, the other paths need dense ones.
struct Strides {
  size_t in_pitch = 0, in_fs = 0, out_pitch = 0, out_fs = 0;
  bool dense() const { return !in_pitch && !in_fs && !out_pitch && !out_fs; }
};

int enqueue_device(sharp_ctx *ctx, const uint8_t *din, int n, int w, int h, const sharp::Params &prm,
                   uint8_t *dout, cudaStream_t st, Slot &slot, size_t chunk, size_t frame_base, int *launches,
                   unsigned int *tc, const Strides &str = Strides(), bool pipelined = false) {
  const size_t fb = (size_t)w * h;
  if (!str.dense() && (ctx->path == SHARP_PATH_STAGED || ctx->path == SHARP_PATH_FUSED || ctx->path == SHARP_PATH_FUSED_EXP))
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "strided frames on the staged / scalar fused paths");
  const size_t nchunks = ((size_t)n + chunk - 1) / chunk;
  if (ctx->path == SHARP_PATH_FUSED || ctx->path == SHARP_PATH_FUSED_EXP) {  // scalar fused ladder rungs
    if (prm.flags & sharp::kReadPerPixel)
      return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "the scalar fused paths implement the default R2 / R5 / R14");
    if ((rc_staged(ctx, slot, st, w, h))) return SHARP_ENOMEM;
    for (int f = 0; f < n; ++f) {
      CK(timed(ctx, st, 2, (double)fb, [&] {
        return sharp::launch_scalar(din + (size_t)f * fb, w, h, prm, slot.staged, ctx->sums + frame_base + f,
                                    ctx->means + frame_base + f, dout + (size_t)f * fb, ctx->path == SHARP_PATH_FUSED,
                                    st);
      }));
      *launches += sharp::kScalarLaunches;
    }
    return SHARP_OK;
  }
  if (ctx->path == SHARP_PATH_STAGED) {  // the paper's base design: K1..K7 per frame
    if ((rc_staged(ctx, slot, st, w, h))) return SHARP_ENOMEM;
    sharp::StageTimer tm;
    if (ctx->profiling) {
      tm.ctx = ctx;
      tm.rec = stage_rec;
    }
    for (int f = 0; f < n; ++f) {
      CK(sharp::launch_staged(din + (size_t)f * fb, w, h, prm, slot.staged, ctx->sums + frame_base + f,
                              ctx->means + frame_base + f, dout + (size_t)f * fb, st, tm));
      *launches += sharp::kStagedLaunches;
    }
    return SHARP_OK;
  }
  // The step kernel implements the LUT-only reading switches; R2 / R5 / R14
  // change per-pixel arithmetic and run on the two-pass path.
  const bool tma_ok = (str.dense() ? sharp::tma_supported(din, dout, w, h)
                                    : sharp::tma_supported_strided(din, str.in_pitch, str.in_fs, dout, str.out_pitch,
                                                                   str.out_fs, w, h)) &&
                      !(prm.flags & sharp::kReadPerPixel);
  if (!str.dense() && !tma_ok) return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "strided frames need the step kernel");
  if (ctx->path == SHARP_PATH_STEP && !tma_ok)
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s",
                   "SHARP_PATH_STEP needs w % 16 == 0, 16-byte aligned input, 8-byte aligned output, w*h <= 2^29 "
                   "and no per-pixel reading switch (R2, R5, R14)");
  const bool tma = tma_family(ctx->path) && tma_ok;
  // the resident kernel (TMEM pEdge) for frames up to ~10 Mpx, else the step kernel
  // AUTO takes the resident kernel where it measured faster than the step
  // kernel: launches of 1 .. 16 Mpx (single images from 1080p to 4K,
  // batches up to ~7 x 1080p), else the step kernel.
  const double px = (double)n * fb;
  // (not for the host pipeline's chunks: its slots' kernels overlap on
  // several streams, which a cooperative launch would serialise)
  const bool res_auto = ctx->path == SHARP_PATH_AUTO && !pipelined && px > kResAutoMinPx && px <= kResAutoMaxPx;
  const bool res = tma && (ctx->path == SHARP_PATH_RES || res_auto) && sharp::res_supported(w, h, n);
  if (ctx->path == SHARP_PATH_RES && !res)
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s",
                   "SHARP_PATH_RES needs the step kernel's geometry and at most 2 x (resident grid) tiles of "
                   "960 x 12 per frame");
  if (tma) {  // the whole batch in one persistent launch
    sharp::BatchLaunch a;
    a.in = din;
    a.n = n;
    a.out = dout;
    a.acc = ctx->acc + frame_base;
    a.sums = ctx->sums + frame_base;
    a.means = ctx->means + frame_base;
    a.luts = ctx->luts + frame_base * sharp::kLutSize;
    a.lut_done = ctx->lut_done + frame_base;
    a.lut_next = ctx->lut_next + frame_base;
    a.task_counter = tc;
    a.in_pitch = str.in_pitch;
    a.in_fs = str.in_fs;
    a.out_pitch = str.out_pitch;
    a.out_fs = str.out_fs;
    CK(timed(ctx, st, 3, (double)n * fb, [&] {
      return res ? sharp::launch_batch_res(a, w, h, prm, st) : sharp::launch_batch_tma(a, w, h, prm, st);
    }));
    *launches += 1;
    return SHARP_OK;
  }
  (void)nchunks;
  for (size_t f0 = 0; f0 < (size_t)n; f0 += chunk) {
    const int cn = (int)std::min(chunk, (size_t)n - f0);
    const double px = (double)cn * fb;
    const uint8_t *ci = din + f0 * fb;
    uint8_t *co = dout + f0 * fb;
    CK(timed(ctx, st, 1, px, [&] {
      return sharp::launch_edge_sum(ci, cn, w, h, prm, ctx->sums + frame_base + f0, slot.counters, slot.luts,
                                    ctx->means + frame_base + f0, st);
    }));
    CK(timed(ctx, st, 2, px, [&] { return sharp::launch_sharpen(ci, cn, w, h, slot.luts, co, prm.flags, st); }));
    *launches += sharp::kLaunchesPerChunk;
  }
  return SHARP_OK;
}

struct Layout {
  size_t pitch, fs;
  int es;
};
int run_general(sharp_ctx *ctx, const uint8_t *in, const Layout &Li, int n, int C, int w, int h,
                const sharp::Params &prm, uint8_t *out, const Layout &Lo, Kind kin, Kind kout);

int run_impl(sharp_ctx *ctx, const uint8_t *in, int n, int w, int h, const sharp_params *pp, uint8_t *out,
             bool async, int flags = 0) {
  int rc = validate(ctx, in, out, n, w, h, pp);
  if (rc) return rc;
  sharp_params p;
  if (pp) p = *pp;
  else sharp_default_params(&p);
  const sharp::Params prm{p.amount, p.gamma, p.osc_gain, p.osc_scale, flags};
  Kind kin, kout;
  if ((rc = classify(ctx, in, &kin)) || (rc = classify(ctx, out, &kout))) return rc;
  if (async && (kin != kDevice || kout != kDevice))
    return set_err(ctx, SHARP_EINVAL, "%s", "sharp_enqueue_batch takes device pointers only");
  if ((kin == kDevice && ((uintptr_t)in & 3)) || (kout == kDevice && ((uintptr_t)out & 3)))
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "device buffers must be 4-byte aligned");
  CK(cudaSetDevice(ctx->device));
  // Device frames with w % 16 == 8 cannot be TMA tensors in place (16-byte
  // row stride): through a 16-byte-pitch scratch they still run on the step
  // kernel (gather + scatter cost 4 B/px, far less than the two-pass path's
  // compute at these widths).  Synchronous calls only.
  if (!async && kin == kDevice && kout == kDevice && (w % 16) == 8 && w >= 24 && !(prm.flags & sharp::kReadPerPixel) &&
      tma_family(ctx->path) && (size_t)w * h <= (1u << 29)) {
    const Layout L{(size_t)w, (size_t)w * h, 1};
    return run_general(ctx, in, L, n, 1, w, h, prm, out, L, kin, kout);
  }
  const auto t0 = std::chrono::steady_clock::now();
  const size_t fb = (size_t)w * h;
  const bool staged = !(kin == kDevice && kout == kDevice);
  // host pipeline whose chunks run on the step kernel (staging buffers are
  // cudaMalloc'd, so only the geometry, the path and the switches decide)
  const bool step_chunks = staged && (w % 16) == 0 && (size_t)w * h <= (1u << 29) &&
                           tma_family(ctx->path) &&
                           !(prm.flags & sharp::kReadPerPixel);
  const size_t chunk = chunk_frames(ctx, fb, n, step_chunks ? kHostStepChunkBudget : kL2ChunkBudget);
  if ((rc = ensure_frames(ctx, (size_t)n))) return rc;
  if ((rc = ensure_slots(ctx, chunk, fb, staged))) return rc;
  int launches = 0;
  const size_t nchunks_all = ((size_t)n + chunk - 1) / chunk;
  if ((rc = ensure_task_counters(ctx, 2 * nchunks_all + 2))) return rc;
  CK(cudaMemsetAsync(ctx->zero_block, 0, ctx->zero_bytes, ctx->stream));  // acc, sums, lut_done, counters
  // (an asynchronous device-resident call reports no device time: no event
  // record between its launches and the previous call's -- measured 2-3 us
  // of a single-image call in a back-to-back stream)
  if (!async || staged) CK(cudaEventRecord(ctx->ev_start, ctx->stream));
  if (!staged) {
    if ((rc = enqueue_device(ctx, in, n, w, h, prm, out, ctx->stream, ctx->slots[0], chunk, 0, &launches,
                             ctx->tcounters)))
      return rc;
  } else {
    // Host pipeline (sec. V-A): chunk c on slot c % nslots; H2D || kernels || D2H.
    const size_t nchunks = ((size_t)n + chunk - 1) / chunk;
    std::vector<size_t> pending_off(ctx->nslots, (size_t)-1), pending_n(ctx->nslots, 0);
    for (int i = 0; i < ctx->nslots; ++i) CK(cudaStreamWaitEvent(ctx->slots[i].stream, ctx->ev_start, 0));
    auto drain = [&](int s) -> int {
      if (pending_off[s] == (size_t)-1) return SHARP_OK;
      CK(cudaEventSynchronize(ctx->slots[s].done));
      if (kout == kPageable) par_memcpy(out + pending_off[s] * fb, ctx->slots[s].h_out, pending_n[s] * fb);
      pending_off[s] = (size_t)-1;
      return SHARP_OK;
    };
    for (size_t c = 0; c < nchunks; ++c) {
      const int s = (int)(c % ctx->nslots);
      Slot &sl = ctx->slots[s];
      if ((rc = drain(s))) return rc;
      const size_t f0 = c * chunk, cn = std::min(chunk, (size_t)n - f0), bytes = cn * fb;
      const uint8_t *src = in + f0 * fb;
      const uint8_t *dsrc = src;
      if (kin != kDevice) {
        if (kin == kPageable) {
          par_memcpy(sl.h_in, src, bytes);
          src = sl.h_in;
        }
        CK(cudaMemcpyAsync(sl.d_in, src, bytes, cudaMemcpyHostToDevice, sl.stream));
        dsrc = sl.d_in;
      }
      uint8_t *ddst = (kout == kDevice) ? out + f0 * fb : sl.d_out;
      if ((rc = enqueue_device(ctx, dsrc, (int)cn, w, h, prm, ddst, sl.stream, sl, cn, f0, &launches,
                               ctx->tcounters + 2 * c, Strides(), true)))
        return rc;
      if (kout != kDevice) {
        uint8_t *hdst = (kout == kPinned) ? out + f0 * fb : sl.h_out;
        CK(cudaMemcpyAsync(hdst, sl.d_out, bytes, cudaMemcpyDeviceToHost, sl.stream));
      }
      CK(cudaEventRecord(sl.done, sl.stream));
      pending_off[s] = f0;
      pending_n[s] = cn;
    }
    for (int s = 0; s < ctx->nslots; ++s) {
      if ((rc = drain(s))) return rc;
      CK(cudaStreamWaitEvent(ctx->stream, ctx->slots[s].done, 0));
    }
  }
  ctx->last_frames = n;
  ctx->stats.frames = n;
  ctx->stats.kernels = launches;
  if (async) return SHARP_OK;
  CK(cudaEventRecord(ctx->ev_stop, ctx->stream));
  // frame 0's S and mean ride on the stream into pinned host memory: one
  // synchronisation per call instead of two more blocking copies
  CK(cudaMemcpyAsync(&ctx->h_stats->sum, ctx->sums, sizeof(unsigned long long), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaMemcpyAsync(&ctx->h_stats->mean, ctx->means, sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  float ms = 0.0f;
  CK(cudaEventElapsedTime(&ms, ctx->ev_start, ctx->ev_stop));
  ctx->stats.edge_sum = ctx->h_stats->sum;
  ctx->stats.edge_mean = ctx->h_stats->mean;
  ctx->stats.device_ms = ms;
  ctx->stats.total_ms =
      std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return SHARP_OK;
}


// ---- General layouts (R1').
bool layout_of(const sharp_layout *l, int w, int h, Layout *o) {
  o->es = (l && l->elem_stride > 0) ? l->elem_stride : 1;
  o->pitch = (l && l->pitch) ? l->pitch : (size_t)w * o->es;
  o->fs = (l && l->frame_stride) ? l->frame_stride : o->pitch * h;
  return o->pitch >= (size_t)w * o->es && o->fs >= o->pitch * (size_t)h;
}

// Bytes from the first to one past the last byte a layout touches.
size_t layout_span(const Layout &L, int n, int C, int w, int h) {
  return (size_t)(n - 1) * L.fs + (size_t)(h - 1) * L.pitch + (size_t)(w - 1) * L.es + (size_t)C;
}

int grow(sharp_ctx *ctx, uint8_t **buf, size_t *cap, size_t need) {
  if (need <= *cap) return SHARP_OK;
  CK(cudaStreamSynchronize(ctx->stream));
  cudaFree(*buf);
  *buf = nullptr;
  *cap = 0;
  CK(cudaMalloc(buf, need));
  *cap = need;
  return SHARP_OK;
}

constexpr size_t kGeneralChunkBytes = 256u << 20;  // dense padded bytes per chunk (each of in / out)

int run_general(sharp_ctx *ctx, const uint8_t *in, const Layout &Li, int n, int C, int w, int h,
                const sharp::Params &prm, uint8_t *out, const Layout &Lo, Kind kin, Kind kout) {
  const int W4 = (w + 3) & ~3, H4 = (h + 3) & ~3;
  // Units whose padded width is a multiple of 8 run on the step kernel from a
  // scratch with a 16-byte row pitch (the TMA stride rule); others dense on
  // the two-pass path.
  const bool step = (W4 % 8) == 0 && W4 >= 16 && H4 >= 8 && tma_family(ctx->path) &&
                    !(prm.flags & sharp::kReadPerPixel) && (size_t)W4 * H4 <= (1u << 29);
  const int P = step ? (W4 + 15) & ~15 : W4;
  const size_t ub = (size_t)P * H4;
  Strides str;
  if (P != W4) str = Strides{(size_t)P, ub, (size_t)P, ub};
  // frames per chunk: sharp_config.chunk_frames if set, else ~kGeneralChunkBytes of padded units
  const int fpc = ctx->chunk_cfg > 0 ? std::min(ctx->chunk_cfg, n)
                                     : (int)std::max<size_t>(1, std::min<size_t>((size_t)n, kGeneralChunkBytes / (ub * C)));
  const size_t units_all = (size_t)n * C;
  int rc;
  if ((rc = ensure_frames(ctx, units_all))) return rc;
  const size_t cu_max = (size_t)fpc * C;
  const size_t chunk = chunk_frames(ctx, ub, (int)cu_max);
  if ((rc = ensure_slots(ctx, chunk, ub, false))) return rc;
  if ((rc = ensure_task_counters(ctx, 2))) return rc;
  if ((rc = grow(ctx, &ctx->gx_in, &ctx->gx_cap, cu_max * ub))) return rc;
  if ((rc = grow(ctx, &ctx->gx_out, &ctx->gx_out_cap, cu_max * ub))) return rc;
  int launches = 0;
  // one memset zeroes every unit's acc / sums / lut_done and the task
  // counters (chunk c uses counter c)
  if ((rc = ensure_task_counters(ctx, (size_t)((n + fpc - 1) / fpc) + 1))) return rc;
  CK(cudaMemsetAsync(ctx->zero_block, 0, ctx->zero_bytes, ctx->stream));
  CK(cudaEventRecord(ctx->ev_start, ctx->stream));
  for (int f0 = 0; f0 < n; f0 += fpc) {
    const int fn = std::min(fpc, n - f0), units = fn * C;
    const size_t u0 = (size_t)f0 * C;
    // source bytes of frames [f0, f0 + fn) on the device
    const uint8_t *src = in + (size_t)f0 * Li.fs;
    if (kin != kDevice) {
      const size_t span = layout_span(Li, fn, C, w, h);
      if ((rc = grow(ctx, &ctx->gx_src, &ctx->gx_src_cap, span))) return rc;
      CK(cudaMemcpyAsync(ctx->gx_src, src, span, cudaMemcpyHostToDevice, ctx->stream));
      src = ctx->gx_src;
    }
    CK(sharp::launch_gather(src, Li.fs, Li.pitch, Li.es, C, w, h, W4, H4, P, units, ctx->gx_in, ctx->stream));
    if ((rc = enqueue_device(ctx, ctx->gx_in, units, W4, H4, prm, ctx->gx_out, ctx->stream, ctx->slots[0],
                             std::min(chunk, (size_t)units), u0, &launches, ctx->tcounters + f0 / fpc, str)))
      return rc;
    // the w x h crops into the caller's layout (a host destination goes
    // through a device copy of its byte range, so bytes between the pixels
    // keep their values)
    uint8_t *dst = out + (size_t)f0 * Lo.fs;
    if (kout == kDevice) {
      CK(sharp::launch_scatter(ctx->gx_out, P, H4, units, w, h, dst, Lo.fs, Lo.pitch, Lo.es, C, ctx->stream));
    } else {
      const size_t span = layout_span(Lo, fn, C, w, h);
      if ((rc = grow(ctx, &ctx->gx_dst, &ctx->gx_dst_cap, span))) return rc;
      CK(cudaMemcpyAsync(ctx->gx_dst, dst, span, cudaMemcpyHostToDevice, ctx->stream));
      CK(sharp::launch_scatter(ctx->gx_out, P, H4, units, w, h, ctx->gx_dst, Lo.fs, Lo.pitch, Lo.es, C,
                               ctx->stream));
      CK(cudaMemcpyAsync(dst, ctx->gx_dst, span, cudaMemcpyDeviceToHost, ctx->stream));
    }
    launches += 2;
    // host byte ranges (pageable or pinned) are reused by the next chunk
    if (kin != kDevice || kout != kDevice) CK(cudaStreamSynchronize(ctx->stream));
  }
  CK(cudaEventRecord(ctx->ev_stop, ctx->stream));
  CK(cudaMemcpyAsync(&ctx->h_stats->sum, ctx->sums, sizeof(unsigned long long), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaMemcpyAsync(&ctx->h_stats->mean, ctx->means, sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  float ms = 0.0f;
  CK(cudaEventElapsedTime(&ms, ctx->ev_start, ctx->ev_stop));
  ctx->last_frames = (int)units_all;
  ctx->stats.frames = (int)units_all;
  ctx->stats.kernels = launches;
  ctx->stats.edge_sum = ctx->h_stats->sum;
  ctx->stats.edge_mean = ctx->h_stats->mean;
  ctx->stats.device_ms = ms;
  ctx->stats.total_ms = ms;
  return SHARP_OK;
}

// Device-resident strided frames straight through the step kernel (no
// copies): an ROI / pitched batch whose strides meet the TMA rules.
int run_device_strided(sharp_ctx *ctx, const uint8_t *in, const Layout &Li, int n, int w, int h,
                       const sharp::Params &prm, uint8_t *out, const Layout &Lo) {
  const auto t0 = std::chrono::steady_clock::now();
  int rc;
  if ((rc = ensure_frames(ctx, (size_t)n))) return rc;
  if ((rc = ensure_slots(ctx, 1, (size_t)w * h, false))) return rc;
  CK(cudaMemsetAsync(ctx->zero_block, 0, ctx->zero_bytes, ctx->stream));
  CK(cudaEventRecord(ctx->ev_start, ctx->stream));
  int launches = 0;
  if ((rc = enqueue_device(ctx, in, n, w, h, prm, out, ctx->stream, ctx->slots[0], (size_t)n, 0, &launches,
                           ctx->tcounters, Strides{Li.pitch, Li.fs, Lo.pitch, Lo.fs})))
    return rc;
  CK(cudaEventRecord(ctx->ev_stop, ctx->stream));
  CK(cudaMemcpyAsync(&ctx->h_stats->sum, ctx->sums, sizeof(unsigned long long), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaMemcpyAsync(&ctx->h_stats->mean, ctx->means, sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  float ms = 0.0f;
  CK(cudaEventElapsedTime(&ms, ctx->ev_start, ctx->ev_stop));
  ctx->last_frames = n;
  ctx->stats.frames = n;
  ctx->stats.kernels = launches;
  ctx->stats.edge_sum = ctx->h_stats->sum;
  ctx->stats.edge_mean = ctx->h_stats->mean;
  ctx->stats.device_ms = ms;
  ctx->stats.total_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return SHARP_OK;
}

int run_ex_impl(sharp_ctx *ctx, const uint8_t *in, const sharp_layout *lin, int n, int C, int w, int h,
                const sharp_params *pp, int flags, uint8_t *out, const sharp_layout *lout) {
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  if (!in || !out) return set_err(ctx, SHARP_EINVAL, "%s", "NULL image pointer");
  if (n < 1 || C < 1) return set_err(ctx, SHARP_EINVAL, "%s", "n < 1 or channels < 1");
  if (w < 5 || h < 5) return set_err(ctx, SHARP_EINVAL, "%s", "width and height must be >= 5 (R1')");
  if (w > 65532 || h > 65532 || (long long)((w + 3) & ~3) * ((h + 3) & ~3) >= (1ll << 31))
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "image larger than 2^31 pixels");
  if (flags & ~sharp::kReadAll) return set_err(ctx, SHARP_EINVAL, "%s", "unknown reading switch");
  if (pp && !params_ok(*pp)) return set_err(ctx, SHARP_EINVAL, "%s", "parameter out of range or not finite");
  Layout Li, Lo;
  if (!layout_of(lin, w, h, &Li) || !layout_of(lout, w, h, &Lo))
    return set_err(ctx, SHARP_EINVAL, "%s", "layout: pitch < w * elem_stride or frame_stride < pitch * h");
  if (C > 1 && (C > Li.es || C > Lo.es))
    return set_err(ctx, SHARP_EINVAL, "%s", "channels > elem_stride (interleaved channels overlap)");
  const bool dense = C == 1 && Li.es == 1 && Lo.es == 1 && Li.pitch == (size_t)w && Lo.pitch == (size_t)w &&
                     Li.fs == (size_t)w * h && Lo.fs == (size_t)w * h && !(w & 3) && !(h & 3) && w >= 8 && h >= 8;
  const uintptr_t a = (uintptr_t)in, b = (uintptr_t)out;
  const size_t sa = layout_span(Li, n, C, w, h), sb = layout_span(Lo, n, C, w, h);
  const bool overlap = a < b + sb && b < a + sa;
  const bool same = a == b && Li.pitch == Lo.pitch && Li.fs == Lo.fs && Li.es == Lo.es;
  if (overlap && !same)
    return set_err(ctx, SHARP_EINVAL, "%s", "input and output overlap without being the same layout (in-place)");
  if (dense && !overlap) return run_impl(ctx, in, n, w, h, pp, out, false, flags);
  sharp_params p;
  if (pp) p = *pp;
  else sharp_default_params(&p);
  const sharp::Params prm{p.amount, p.gamma, p.osc_gain, p.osc_scale, flags};
  Kind kin, kout;
  int rc;
  if ((rc = classify(ctx, in, &kin)) || (rc = classify(ctx, out, &kout))) return rc;
  CK(cudaSetDevice(ctx->device));
  // zero-copy: single-channel device frames with w % 8 == 0, h % 4 == 0 and
  // strides the TMA step kernel takes directly
  if (C == 1 && Li.es == 1 && Lo.es == 1 && !overlap && kin == kDevice && kout == kDevice && !(w & 7) && !(h & 3) &&
      w >= 8 && h >= 8 && tma_family(ctx->path) &&
      !(flags & sharp::kReadPerPixel) &&
      sharp::tma_supported_strided(in, Li.pitch, Li.fs, out, Lo.pitch, Lo.fs, w, h))
    return run_device_strided(ctx, in, Li, n, w, h, prm, out, Lo);
  return run_general(ctx, in, Li, n, C, w, h, prm, out, Lo, kin, kout);
}

// Row bands (sec. 8(e) of SURVEY.md / DESIGN.md sec. 9).
int band_halo(int h, int row0, int row1, int *in0, int *in1) {
  if (h < 8 || (h & 3) || row0 < 0 || row1 > h || row0 >= row1 || (row0 & 3) || (row1 & 3)) return SHARP_EINVAL;
  *in0 = std::max(row0 - 4, 0);
  *in1 = std::min(row1 + 4, h);
  return SHARP_OK;
}

int band_impl(sharp_ctx *ctx, int mode, const uint8_t *band, int w, int h, int row0, int row1,
              unsigned long long *partial, const unsigned long long *total, const sharp_params *pp, uint8_t *out) {
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  int in0 = 0, in1 = 0;
  if (!band || (mode == sharp::kStepPass1 ? !partial : (!total || !out)))
    return set_err(ctx, SHARP_EINVAL, "%s", "NULL pointer");
  if (w < 8 || (w & 3) || band_halo(h, row0, row1, &in0, &in1))
    return set_err(ctx, SHARP_EINVAL, "%s", "bad band geometry (multiples of 4, 0 <= row0 < row1 <= h)");
  if ((long long)w * h >= (1ll << 29) || w > 65536 || h > 65536)
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "image larger than 2^29 pixels");
  if (pp && !params_ok(*pp)) return set_err(ctx, SHARP_EINVAL, "%s", "parameter out of range or not finite");
  Kind k;
  int rc;
  if ((rc = classify(ctx, band, &k))) return rc;
  if (k != kDevice) return set_err(ctx, SHARP_EINVAL, "%s", "band calls take device pointers only");
  if (mode == sharp::kStepPass2) {
    if ((rc = classify(ctx, out, &k))) return rc;
    if (k != kDevice) return set_err(ctx, SHARP_EINVAL, "%s", "band calls take device pointers only");
    const uintptr_t a = (uintptr_t)band, b = (uintptr_t)out;
    const size_t na = (size_t)(in1 - in0) * w, nb = (size_t)(row1 - row0) * w;
    if (a < b + nb && b < a + na) return set_err(ctx, SHARP_EINVAL, "%s", "input and output overlap");
  }
  if (!tma_family(ctx->path) ||
      !sharp::tma_supported(band, mode == sharp::kStepPass2 ? out : (uint8_t *)band, w, h))
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s",
                   "row bands need the TMA path (w % 16 == 0, 16-byte aligned band, 8-byte aligned out)");
  sharp_params p;
  if (pp) p = *pp;
  else sharp_default_params(&p);
  const sharp::Params prm{p.amount, p.gamma, p.osc_gain, p.osc_scale};
  CK(cudaSetDevice(ctx->device));
  if ((rc = ensure_frames(ctx, 1))) return rc;
  if ((rc = ensure_task_counters(ctx, 1))) return rc;
  sharp::BatchLaunch a;
  a.in = band;
  a.n = 1;
  a.out = out;
  a.acc = ctx->acc;
  a.sums = ctx->sums;
  a.means = ctx->means;
  a.luts = ctx->luts;
  a.lut_done = ctx->lut_done;
  a.task_counter = ctx->tcounters;
  a.partial = partial;
  a.total = total;
  if (mode == sharp::kStepPass1) {
    CK(cudaMemsetAsync(ctx->acc, 0, sizeof(unsigned long long), ctx->stream));
    CK(cudaMemsetAsync(ctx->tcounters, 0, sizeof(unsigned int), ctx->stream));
  }
  const double px = (double)(row1 - row0) * w;
  CK(timed(ctx, ctx->stream, mode == sharp::kStepPass1 ? 1 : 2, px, [&] {
    return sharp::launch_band_tma(a, mode, w, h, row0, row1, in0, in1 - in0, prm, ctx->stream);
  }));
  ctx->last_frames = 1;
  ctx->stats.frames = 1;
  ctx->stats.kernels = 2;
  return SHARP_OK;
}

// ---- Multi-device contexts (sharp_config.num_devices > 1).
bool is_multi(const sharp_ctx *c) { return c && !c->sub.empty(); }

int band_rows_of(int h, int G, int g, int *r0, int *r1) {
  if (h < 8 || (h & 3) || G < 1 || g < 0 || g >= G || h / 4 < G) return SHARP_EINVAL;
  const int blocks = h / 4, base = blocks / G, rem = blocks % G;
  const int start = g * base + std::min(g, rem), count = base + (g < rem ? 1 : 0);
  *r0 = 4 * start;
  *r1 = 4 * (start + count);
  return SHARP_OK;
}

// Copies a sub-context's failure into the multi context.
int sub_fail(sharp_ctx *m, int g, int rc) {
  if (rc != SHARP_OK) snprintf(m->err, sizeof(m->err), "device %d (entry %d): %s", m->sub[g]->device, g, m->sub[g]->err);
  return rc;
}

int grow_dev(sharp_ctx *sc, uint8_t **buf, size_t *cap, size_t need) {
  if (need <= *cap) return SHARP_OK;
  cudaSetDevice(sc->device);
  cudaStreamSynchronize(sc->stream);
  cudaFree(*buf);
  *buf = nullptr;
  *cap = 0;
  if (cudaMalloc(buf, need) != cudaSuccess) {
    cudaGetLastError();
    return SHARP_ENOMEM;
  }
  *cap = need;
  return SHARP_OK;
}

// Frames split over the devices: contiguous ranges, one
// thread per device (each sub-context is used by one thread), host buffers.
int multi_frames(sharp_ctx *m, const uint8_t *in, int n, int w, int h, const sharp_params *pp, uint8_t *out) {
  const int G = (int)m->sub.size();
  const size_t fb = (size_t)w * h;
  const auto t0 = std::chrono::steady_clock::now();
  m->last_split.assign(G, {0, 0});
  std::vector<int> rc(G, SHARP_OK);
  std::vector<std::thread> th;
  for (int g = 0; g < G; ++g) {
    const int base = n / G, rem = n % G, f0 = g * base + std::min(g, rem), cnt = base + (g < rem ? 1 : 0);
    m->last_split[g] = {f0, cnt};
    if (cnt == 0) continue;
    th.emplace_back([=, &rc] { rc[g] = run_impl(m->sub[g], in + (size_t)f0 * fb, cnt, w, h, pp, out + (size_t)f0 * fb, false); });
  }
  for (auto &t : th) t.join();
  m->stats = sharp_stats{};
  for (int g = 0; g < G; ++g) {
    if (rc[g] != SHARP_OK) return sub_fail(m, g, rc[g]);
    if (m->last_split[g].second == 0) continue;
    const sharp_stats &st = m->sub[g]->stats;
    if (m->last_split[g].first == 0) {
      m->stats.edge_sum = st.edge_sum;
      m->stats.edge_mean = st.edge_mean;
    }
    m->stats.device_ms = std::max(m->stats.device_ms, st.device_ms);
    m->stats.kernels += st.kernels;
  }
  m->stats.frames = n;
  m->last_frames = n;
  m->stats.total_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return SHARP_OK;
}

// One image as G row bands, one per device: each band's rows
// with their 4-row halos go to the band's device (from the host image, or
// from the neighbouring device bands by peer copies), pass 1 sums pEdge over
// the band's rows, the G partials are added (the L174 mean), pass 2 writes
// the band.  `bands` == nullptr: `img`/`out` are host images; else device
// bands / outputs per device (sharp_run_bands).
int multi_rows(sharp_ctx *m, const uint8_t *img, const uint8_t *const *bands, int w, int h, const sharp_params *pp,
               uint8_t *out, uint8_t *const *outs) {
  const int G = (int)m->sub.size();
  const auto t0 = std::chrono::steady_clock::now();
  if (w < 16 || (w & 15) || h < 8 || (h & 3) || h / 4 < G)
    return set_err(m, SHARP_EUNSUPPORTED, "%s", "row bands need w % 16 == 0, h % 4 == 0 and >= 4 rows per band");
  if (pp && !params_ok(*pp)) return set_err(m, SHARP_EINVAL, "%s", "parameter out of range or not finite");
  std::vector<int> r0(G), r1(G), i0(G), i1(G);
  for (int g = 0; g < G; ++g) {
    band_rows_of(h, G, g, &r0[g], &r1[g]);
    band_halo(h, r0[g], r1[g], &i0[g], &i1[g]);
  }
  int rc;
  for (int g = 0; g < G; ++g) {  // stage each band + halos on its device, pass 1
    sharp_ctx *sc = m->sub[g];
    sharp_ctx::BandBuf &b = m->bb[g];
    const size_t in_bytes = (size_t)(i1[g] - i0[g]) * w, own = (size_t)(r1[g] - r0[g]) * w;
    if ((rc = grow_dev(sc, &b.in, &b.in_cap, in_bytes)) || (!bands && (rc = grow_dev(sc, &b.out, &b.out_cap, own))))
      return set_err(m, rc, "%s", "band scratch allocation failed");
    if (cudaSetDevice(sc->device) != cudaSuccess) return set_err(m, SHARP_ECUDA, "%s", "cudaSetDevice");
    cudaError_t e = cudaSuccess;
    if (!bands) {
      e = cudaMemcpyAsync(b.in, img + (size_t)i0[g] * w, in_bytes, cudaMemcpyHostToDevice, sc->stream);
    } else {
      uint8_t *dst = b.in + (size_t)(r0[g] - i0[g]) * w;
      e = cudaMemcpyAsync(dst, bands[g], own, cudaMemcpyDeviceToDevice, sc->stream);  // own rows
      if (e == cudaSuccess && g > 0)  // upper halo: the last r0 - i0 rows of band g-1
        e = cudaMemcpyPeerAsync(b.in, sc->device, bands[g - 1] + (size_t)(i0[g] - r0[g - 1]) * w,
                                m->sub[g - 1]->device, (size_t)(r0[g] - i0[g]) * w, sc->stream);
      if (e == cudaSuccess && g + 1 < G)  // lower halo: the first i1 - r1 rows of band g+1
        e = cudaMemcpyPeerAsync(b.in + (size_t)(r1[g] - i0[g]) * w, sc->device, bands[g + 1],
                                m->sub[g + 1]->device, (size_t)(i1[g] - r1[g]) * w, sc->stream);
    }
    if (e != cudaSuccess) return set_err(m, SHARP_ECUDA, "band copy: %s", cudaGetErrorString(e));
    if ((rc = band_impl(sc, sharp::kStepPass1, b.in, w, h, r0[g], r1[g], b.part, nullptr, nullptr, nullptr)))
      return sub_fail(m, g, rc);
    if ((e = cudaMemcpyAsync(&b.h[0], b.part, 8, cudaMemcpyDeviceToHost, sc->stream)) != cudaSuccess)
      return set_err(m, SHARP_ECUDA, "partial D2H: %s", cudaGetErrorString(e));
  }
  unsigned long long S = 0;  // L174: the sum over the whole image
  for (int g = 0; g < G; ++g) {
    cudaSetDevice(m->sub[g]->device);
    if (cudaStreamSynchronize(m->sub[g]->stream) != cudaSuccess) return set_err(m, SHARP_ECUDA, "%s", "band pass 1");
    S += m->bb[g].h[0];
  }
  for (int g = 0; g < G; ++g) {  // pass 2 with the all-reduced S
    sharp_ctx *sc = m->sub[g];
    sharp_ctx::BandBuf &b = m->bb[g];
    cudaSetDevice(sc->device);
    b.h[1] = S;
    cudaError_t e = cudaMemcpyAsync(b.total, &b.h[1], 8, cudaMemcpyHostToDevice, sc->stream);
    if (e != cudaSuccess) return set_err(m, SHARP_ECUDA, "total H2D: %s", cudaGetErrorString(e));
    uint8_t *dst = bands ? outs[g] : b.out;
    if ((rc = band_impl(sc, sharp::kStepPass2, b.in, w, h, r0[g], r1[g], nullptr, b.total, pp, dst)))
      return sub_fail(m, g, rc);
    if (!bands && (e = cudaMemcpyAsync(out + (size_t)r0[g] * w, b.out, (size_t)(r1[g] - r0[g]) * w,
                                       cudaMemcpyDeviceToHost, sc->stream)) != cudaSuccess)
      return set_err(m, SHARP_ECUDA, "band D2H: %s", cudaGetErrorString(e));
  }
  for (int g = 0; g < G; ++g) {
    cudaSetDevice(m->sub[g]->device);
    if (cudaStreamSynchronize(m->sub[g]->stream) != cudaSuccess) return set_err(m, SHARP_ECUDA, "%s", "band pass 2");
  }
  m->stats = sharp_stats{};
  m->stats.edge_sum = S;
  m->stats.edge_mean = (double)S / ((double)w * (double)h);  // R8 (sharp_run: default readings)
  m->stats.frames = 1;
  m->stats.kernels = 4 * G;
  m->last_frames = 1;
  m->last_split.assign(1, {0, 1});
  m->stats.total_ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
  m->stats.device_ms = m->stats.total_ms;
  return SHARP_OK;
}

// Host buffers only (the sub-contexts classify the pointers themselves).
int multi_host_check(sharp_ctx *m, const void *a, const void *b) {
  cudaPointerAttributes at;
  for (const void *p : {a, b}) {
    if (cudaPointerGetAttributes(&at, p) == cudaSuccess &&
        (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged))
      return set_err(m, SHARP_EUNSUPPORTED, "%s",
                     "multi-device contexts take host buffers (device-resident bands: sharp_run_bands)");
    cudaGetLastError();
  }
  return SHARP_OK;
}

int multi_run(sharp_ctx *m, const uint8_t *in, int n, int w, int h, const sharp_params *pp, uint8_t *out) {
  if (m->poisoned) return SHARP_ESTATE;
  if (!in || !out || n < 1) return set_err(m, SHARP_EINVAL, "%s", "NULL image pointer or n < 1");
  if (w < 8 || h < 8 || (w & 3) || (h & 3))
    return set_err(m, SHARP_EINVAL, "%s", "width and height must be multiples of 4 and >= 8 (R1)");
  const size_t bytes = (size_t)n * w * h;
  if ((uintptr_t)in < (uintptr_t)out + bytes && (uintptr_t)out < (uintptr_t)in + bytes)
    return set_err(m, SHARP_EINVAL, "%s", "input and output overlap");
  int rc;
  if ((rc = multi_host_check(m, in, out))) return rc;
  const int shard = m->shard == SHARP_SHARD_AUTO ? (n >= 2 ? SHARP_SHARD_FRAMES : SHARP_SHARD_ROWS) : m->shard;
  if (shard == SHARP_SHARD_NONE) {  // everything on the first device
    rc = run_impl(m->sub[0], in, n, w, h, pp, out, false);
    if (rc) return sub_fail(m, 0, rc);
    m->stats = m->sub[0]->stats;
    m->last_frames = n;
    m->last_split.assign(m->sub.size(), {0, 0});
    m->last_split[0] = {0, n};
    return SHARP_OK;
  }
  if (shard == SHARP_SHARD_ROWS) {
    if (n != 1) return set_err(m, SHARP_EUNSUPPORTED, "%s", "SHARP_SHARD_ROWS shards one image (n == 1)");
    return multi_rows(m, in, nullptr, w, h, pp, out, nullptr);
  }
  return multi_frames(m, in, n, w, h, pp, out);
}

#define NOT_MULTI(ctx)                                                                                       \
  do {                                                                                                       \
    if (is_multi(ctx))                                                                                       \
      return set_err(ctx, SHARP_EUNSUPPORTED, "%s",                                                          \
                     "not available on a multi-device context (sharp_run / sharp_run_batch / sharp_run_bands)"); \
  } while (0)

}  // namespace

extern "C" {

int sharp_band_rows(int h, int n_bands, int band, int *row0, int *row1) {
  if (!row0 || !row1) return SHARP_EINVAL;
  return band_rows_of(h, n_bands, band, row0, row1);
}

int sharp_run_bands(sharp_ctx *ctx, const uint8_t *const *bands, int w, int h, const sharp_params *params,
                    uint8_t *const *outs) {
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  if (!bands || !outs) return set_err(ctx, SHARP_EINVAL, "%s", "NULL band array");
  const int G = is_multi(ctx) ? (int)ctx->sub.size() : 1;
  for (int g = 0; g < G; ++g)
    if (!bands[g] || !outs[g]) return set_err(ctx, SHARP_EINVAL, "%s", "NULL band pointer");
  if (G == 1) return run_impl(ctx, bands[0], 1, w, h, params, outs[0], false);
  return multi_rows(ctx, nullptr, bands, w, h, params, nullptr, outs);
}

int sharp_band_halo(int h, int row0, int row1, int *in0, int *in1) {
  if (!in0 || !in1) return SHARP_EINVAL;
  return band_halo(h, row0, row1, in0, in1);
}

int sharp_band_edge_sum(sharp_ctx *ctx, const uint8_t *band, int w, int h, int row0, int row1,
                        uint64_t *d_partial) {
  NOT_MULTI(ctx);
  return band_impl(ctx, sharp::kStepPass1, band, w, h, row0, row1, (unsigned long long *)d_partial, nullptr,
                   nullptr, nullptr);
}

int sharp_band_sharpen(sharp_ctx *ctx, const uint8_t *band, int w, int h, int row0, int row1,
                       const uint64_t *d_total, const sharp_params *params, uint8_t *out) {
  NOT_MULTI(ctx);
  return band_impl(ctx, sharp::kStepPass2, band, w, h, row0, row1, nullptr,
                   (const unsigned long long *)d_total, params, out);
}

void sharp_default_params(sharp_params *p) {
  if (!p) return;
  p->amount = 1.0f;    // R16
  p->gamma = 0.5f;
  p->osc_gain = 0.5f;
  p->osc_scale = 2.0f;
}

int sharp_create(sharp_ctx **out, const sharp_config *cfg) {
  if (!out) return SHARP_EINVAL;
  *out = nullptr;
  sharp_config c{};
  c.device = -1;
  if (cfg) c = *cfg;
  if (c.streams < 0 || c.streams > kMaxSlots || c.chunk_frames < 0 || c.max_frames < 0) return SHARP_EINVAL;
  if (c.num_devices < 0 || c.num_devices > 64 || c.shard < SHARP_SHARD_AUTO || c.shard > SHARP_SHARD_FRAMES)
    return SHARP_EINVAL;
  if (c.num_devices > 1) {  // one single-device context per entry
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess) {
      cudaGetLastError();
      return SHARP_ECUDA;
    }
    sharp_ctx *m = new (std::nothrow) sharp_ctx();
    if (!m) return SHARP_ENOMEM;
    m->shard = c.shard;
    m->device = c.device_ids ? c.device_ids[0] : 0;
    m->bb.resize(c.num_devices);
    for (int g = 0; g < c.num_devices; ++g) {
      const int dev = c.device_ids ? c.device_ids[g] : g;
      sharp_config cs = c;
      cs.num_devices = 0;
      cs.device_ids = nullptr;
      cs.device = dev;
      sharp_ctx *sc = nullptr;
      int rc = (dev < 0 || dev >= ndev) ? SHARP_EINVAL : sharp_create(&sc, &cs);
      if (rc == SHARP_OK) {
        m->sub.push_back(sc);
        sharp_ctx::BandBuf &b = m->bb[g];
        cudaSetDevice(dev);
        if (cudaMalloc(&b.part, 16) != cudaSuccess || cudaHostAlloc(&b.h, 16, cudaHostAllocDefault) != cudaSuccess)
          rc = SHARP_ENOMEM;
        else
          b.total = b.part + 1;
      }
      if (rc != SHARP_OK) {
        cudaGetLastError();
        sharp_destroy(m);
        return rc;
      }
    }
    // peer access between neighbouring devices (the band halo copies); the
    // copies also work without it (staged by the driver)
    for (int g = 0; g + 1 < c.num_devices; ++g) {
      const int a = m->sub[g]->device, b = m->sub[g + 1]->device;
      int ok = 0;
      if (a != b && cudaDeviceCanAccessPeer(&ok, a, b) == cudaSuccess && ok) {
        cudaSetDevice(a);
        cudaDeviceEnablePeerAccess(b, 0);
        cudaSetDevice(b);
        cudaDeviceEnablePeerAccess(a, 0);
      }
      cudaGetLastError();  // (already enabled is fine)
    }
    *out = m;
    return SHARP_OK;
  }
  sharp_ctx *ctx = new (std::nothrow) sharp_ctx();
  if (!ctx) return SHARP_ENOMEM;
  int dev = c.device;
  cudaError_t e = cudaSuccess;
  if (dev < 0) e = cudaGetDevice(&dev);
  int ndev = 0;
  if (e == cudaSuccess) e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || dev >= ndev) {
    cudaGetLastError();
    delete ctx;
    return e != cudaSuccess ? SHARP_ECUDA : SHARP_EINVAL;
  }
  ctx->device = dev;
  {
    const char *g = getenv("SHARP_FORCE_GENERIC");
    ctx->path = (g && g[0] == '1') ? SHARP_PATH_TWO_PASS : SHARP_PATH_AUTO;
  }
  ctx->nslots = c.streams ? c.streams : 3;
  ctx->chunk_cfg = c.chunk_frames;
  int rc = SHARP_OK;
  do {
    if ((e = cudaSetDevice(dev)) != cudaSuccess) break;
    if ((e = cudaStreamCreateWithFlags(&ctx->own_stream, cudaStreamNonBlocking)) != cudaSuccess) break;
    ctx->stream = ctx->own_stream;
    if ((e = cudaEventCreate(&ctx->ev_start)) != cudaSuccess) break;
    if ((e = cudaEventCreate(&ctx->ev_stop)) != cudaSuccess) break;
    if ((e = cudaHostAlloc(&ctx->h_stats, sizeof(*ctx->h_stats), cudaHostAllocDefault)) != cudaSuccess) break;
    for (int i = 0; i < ctx->nslots && e == cudaSuccess; ++i) {
      e = cudaStreamCreateWithFlags(&ctx->slots[i].stream, cudaStreamNonBlocking);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->slots[i].done, cudaEventDisableTiming);
    }
    if (e != cudaSuccess) break;
    // load every kernel now (lazy module loading can deadlock spinning kernels, kernels.h)
    if ((e = sharp::preload_step()) != cudaSuccess || (e = sharp::preload_res()) != cudaSuccess || (e = sharp::preload_two_pass()) != cudaSuccess ||
        (e = sharp::preload_staged()) != cudaSuccess || (e = sharp::preload_scalar()) != cudaSuccess || (e = sharp::preload_p2p()) != cudaSuccess ||
        (e = sharp::preload_layout()) != cudaSuccess)
      break;
    if (c.max_frames > 0 && (rc = ensure_frames(ctx, (size_t)c.max_frames))) break;
    if (c.max_width > 0 && c.max_height > 0) {
      const size_t fb = (size_t)c.max_width * c.max_height;
      if ((rc = ensure_slots(ctx, chunk_frames(ctx, fb, c.max_frames > 0 ? c.max_frames : 1), fb, false))) break;
    }
  } while (0);
  if (e != cudaSuccess || rc != SHARP_OK) {
    cudaGetLastError();
    sharp_destroy(ctx);
    return rc ? rc : (e == cudaErrorMemoryAllocation ? SHARP_ENOMEM : SHARP_ECUDA);
  }
  *out = ctx;
  return SHARP_OK;
}

void sharp_destroy(sharp_ctx *ctx) {
  if (!ctx) return;
  if (!ctx->bb.empty()) {  // multi-device context
    for (size_t g = 0; g < ctx->bb.size(); ++g) {
      sharp_ctx::BandBuf &b = ctx->bb[g];
      if (g < ctx->sub.size()) cudaSetDevice(ctx->sub[g]->device);
      cudaFree(b.in);
      cudaFree(b.out);
      cudaFree(b.part);
      if (b.h) cudaFreeHost(b.h);
    }
    for (sharp_ctx *sc : ctx->sub) sharp_destroy(sc);
    cudaGetLastError();
    delete ctx;
    return;
  }
  cudaSetDevice(ctx->device);
  if (ctx->stream) cudaStreamSynchronize(ctx->stream);
  for (int i = 0; i < kMaxSlots; ++i) {
    Slot &s = ctx->slots[i];
    if (s.stream) cudaStreamSynchronize(s.stream);
    free_slot(s);
    if (s.done) cudaEventDestroy(s.done);
    if (s.stream) cudaStreamDestroy(s.stream);
  }
  cudaFree(ctx->zero_block);
  cudaFree(ctx->means);
  cudaFree(ctx->luts);
  cudaFree(ctx->gx_in);
  cudaFree(ctx->gx_out);
  cudaFree(ctx->gx_src);
  cudaFree(ctx->gx_dst);
  for (auto &r : ctx->recs) {
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  for (auto e : ctx->ev_pool) cudaEventDestroy(e);
  if (ctx->ev_start) cudaEventDestroy(ctx->ev_start);
  if (ctx->ev_stop) cudaEventDestroy(ctx->ev_stop);
  if (ctx->h_stats) cudaFreeHost(ctx->h_stats);
  if (ctx->own_stream) cudaStreamDestroy(ctx->own_stream);
  cudaGetLastError();
  delete ctx;
}

int sharp_set_stream(sharp_ctx *ctx, void *stream) {
  if (!ctx) return SHARP_EINVAL;
  NOT_MULTI(ctx);
  if (ctx->poisoned) return SHARP_ESTATE;
  cudaStream_t next = stream ? (cudaStream_t)stream : ctx->own_stream;
  if (next != ctx->stream) {
    // work already queued on the old stream (a persistent launch, the scratch
    // it uses) completes before anything issued on the new one
    CK(cudaSetDevice(ctx->device));
    cudaEvent_t e = pool_event(ctx);
    if (!e) return set_err(ctx, SHARP_ECUDA, "%s", "cudaEventCreate failed");
    CK(cudaEventRecord(e, ctx->stream));
    CK(cudaStreamWaitEvent(next, e, 0));
    ctx->ev_pool.push_back(e);
  }
  ctx->stream = next;
  return SHARP_OK;
}

int sharp_run(sharp_ctx *ctx, const uint8_t *img, int w, int h, const sharp_params *params, uint8_t *out) {
  if (is_multi(ctx)) return multi_run(ctx, img, 1, w, h, params, out);
  return run_impl(ctx, img, 1, w, h, params, out, false);
}

int sharp_run_batch(sharp_ctx *ctx, const uint8_t *imgs, int n, int w, int h, const sharp_params *params,
                    uint8_t *outs) {
  if (is_multi(ctx)) return multi_run(ctx, imgs, n, w, h, params, outs);
  return run_impl(ctx, imgs, n, w, h, params, outs, false);
}

int sharp_enqueue_batch(sharp_ctx *ctx, const uint8_t *d_imgs, int n, int w, int h, const sharp_params *params,
                        uint8_t *d_outs) {
  NOT_MULTI(ctx);
  return run_impl(ctx, d_imgs, n, w, h, params, d_outs, true);
}

int sharp_run_ex(sharp_ctx *ctx, const uint8_t *imgs, const sharp_layout *in_layout, int n, int channels, int w,
                 int h, const sharp_params *params, int flags, uint8_t *outs, const sharp_layout *out_layout) {
  NOT_MULTI(ctx);
  return run_ex_impl(ctx, imgs, in_layout, n, channels, w, h, params, flags, outs, out_layout);
}

int sharp_get_stats(const sharp_ctx *ctx, sharp_stats *s) {
  if (!ctx || !s) return SHARP_EINVAL;
  *s = ctx->stats;
  return SHARP_OK;
}

int sharp_get_batch_sums(sharp_ctx *ctx, uint64_t *sums, int n) {
  if (!ctx || !sums || n < 0) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  if (n > ctx->last_frames) return set_err(ctx, SHARP_EINVAL, "%s", "n exceeds the frames of the last call");
  if (n == 0) return SHARP_OK;
  if (is_multi(ctx)) {  // gathered from the devices' frame ranges
    if (ctx->last_split.size() == 1) {  // one row-sharded image
      sums[0] = ctx->stats.edge_sum;
      return SHARP_OK;
    }
    for (size_t g = 0; g < ctx->last_split.size(); ++g) {
      const int f0 = ctx->last_split[g].first, cnt = std::min(ctx->last_split[g].second, n - f0);
      if (cnt <= 0) continue;
      const int rc = sharp_get_batch_sums(ctx->sub[g], sums + f0, cnt);
      if (rc) return sub_fail(ctx, (int)g, rc);
    }
    return SHARP_OK;
  }
  CK(cudaStreamSynchronize(ctx->stream));
  CK(cudaMemcpy(sums, ctx->sums, (size_t)n * sizeof(uint64_t), cudaMemcpyDeviceToHost));
  return SHARP_OK;
}

int sharp_set_profiling(sharp_ctx *ctx, int enable) {
  if (!ctx) return SHARP_EINVAL;
  NOT_MULTI(ctx);
  if (ctx->poisoned) return SHARP_ESTATE;
  CK(cudaStreamSynchronize(ctx->stream));
  for (auto &r : ctx->recs) {
    ctx->ev_pool.push_back(r.a);
    ctx->ev_pool.push_back(r.b);
  }
  ctx->recs.clear();
  ctx->profiling = enable != 0;
  return SHARP_OK;
}

int sharp_get_kernel_times(sharp_ctx *ctx, sharp_kernel_times *t) {
  if (!ctx || !t) return SHARP_EINVAL;
  NOT_MULTI(ctx);
  if (ctx->poisoned) return SHARP_ESTATE;
  *t = sharp_kernel_times{};
  for (auto &r : ctx->recs) {
    CK(cudaEventSynchronize(r.b));
    float ms = 0.0f;
    CK(cudaEventElapsedTime(&ms, r.a, r.b));
    if (r.kind == 1) {
      t->pass1_ms += ms;
      t->pass1_launches++;
    } else if (r.kind == 2) {
      t->pass2_ms += ms;
      t->pass2_launches++;
      t->pixels += r.px;
    } else if (r.kind == 3) {
      t->step_ms += ms;
      t->step_launches++;
      t->pixels += r.px;
    }
  }
  return SHARP_OK;
}

int sharp_get_stage_times(sharp_ctx *ctx, float *ms, int n) {
  if (!ctx || !ms || n < SHARP_NUM_STAGES) return SHARP_EINVAL;
  NOT_MULTI(ctx);
  if (ctx->poisoned) return SHARP_ESTATE;
  for (int i = 0; i < SHARP_NUM_STAGES; ++i) ms[i] = 0.0f;
  for (auto &r : ctx->recs) {
    if (r.kind < 10 || r.kind >= 10 + SHARP_NUM_STAGES) continue;
    CK(cudaEventSynchronize(r.b));
    float t = 0.0f;
    CK(cudaEventElapsedTime(&t, r.a, r.b));
    ms[r.kind - 10] += t;
  }
  return SHARP_OK;
}

// ---- fused peer-memory band exchange (bands_p2p.cu)
size_t sharp_p2p_window_bytes(int w, int rows_own) {
  if (w < 16 || (w & 15) || rows_own < 4) return 0;
  return sharp::p2p_window_bytes(w, rows_own);
}

int sharp_p2p_window_create(int w, int rows_own, void **d_window) {
  if (!d_window) return SHARP_EINVAL;
  *d_window = nullptr;
  const size_t bytes = sharp_p2p_window_bytes(w, rows_own);
  if (!bytes) return SHARP_EINVAL;
  if (cudaMalloc(d_window, bytes) != cudaSuccess) {
    cudaGetLastError();
    *d_window = nullptr;
    return SHARP_ENOMEM;
  }
  if (cudaMemset(*d_window, 0, bytes) != cudaSuccess) {
    cudaGetLastError();
    cudaFree(*d_window);
    *d_window = nullptr;
    return SHARP_ECUDA;
  }
  return SHARP_OK;
}

void sharp_p2p_window_destroy(void *d_window) {
  if (d_window) cudaFree(d_window);
}

int sharp_band_p2p_halo(sharp_ctx *ctx, uint8_t *self_window, int w, int rows_own, uint8_t *up_window,
                        int up_rows_own, uint8_t *down_window, uint64_t epoch) {
  NOT_MULTI(ctx);
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  if (!self_window || w < 16 || (w & 15) || rows_own < 4 || epoch == 0 || (up_window && up_rows_own < 4) ||
      (((uintptr_t)self_window | (uintptr_t)up_window | (uintptr_t)down_window) & 15))
    return set_err(ctx, SHARP_EINVAL, "%s", "bad p2p halo request (w % 16, rows >= 4, 16-byte windows, epoch > 0)");
  CK(sharp::launch_p2p_halo(self_window, w, rows_own, up_window, up_rows_own, down_window, epoch, ctx->stream));
  return SHARP_OK;
}

static int band_fused_impl(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank, int w, int h, int row0,
                           int row1, int up_rows_own, bool halo, uint64_t epoch, const sharp_params *params,
                           uint8_t *out, int grid_cap);

int sharp_band_p2p_sharpen(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank, int w, int h, int row0,
                           int row1, uint64_t epoch, const sharp_params *params, uint8_t *out, int grid_cap) {
  NOT_MULTI(ctx);
  return band_fused_impl(ctx, windows, n_ranks, rank, w, h, row0, row1, 0, false, epoch, params, out, grid_cap);
}

int sharp_band_p2p_step(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank, int w, int h, int row0,
                        int row1, int up_rows_own, uint64_t epoch, const sharp_params *params, uint8_t *out,
                        int grid_cap) {
  NOT_MULTI(ctx);
  if (rank > 0 && up_rows_own < 4)
    return ctx ? set_err(ctx, SHARP_EINVAL, "%s", "up_rows_own < 4") : SHARP_EINVAL;
  return band_fused_impl(ctx, windows, n_ranks, rank, w, h, row0, row1, up_rows_own, true, epoch, params, out,
                         grid_cap);
}

static int band_fused_impl(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank, int w, int h, int row0,
                           int row1, int up_rows_own, bool halo, uint64_t epoch, const sharp_params *params,
                           uint8_t *out, int grid_cap) {
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  int in0 = 0, in1 = 0;
  if (!windows || !out || n_ranks < 1 || n_ranks > sharp::kMaxRanks || rank < 0 || rank >= n_ranks || epoch == 0 ||
      grid_cap < 0)
    return set_err(ctx, SHARP_EINVAL, "%s", "bad fused band request (1 <= n_ranks <= 32, epoch > 0)");
  for (int g = 0; g < n_ranks; ++g)
    if (!windows[g] || ((uintptr_t)windows[g] & 15)) return set_err(ctx, SHARP_EINVAL, "%s", "bad window pointer");
  if (w < 16 || (w & 15) || band_halo(h, row0, row1, &in0, &in1) || row1 - row0 < 4)
    return set_err(ctx, SHARP_EINVAL, "%s", "bad band geometry (w % 16 == 0, rows multiples of 4, >= 4 rows)");
  if ((long long)w * h >= (1ll << 29)) return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "image larger than 2^29 pixels");
  if (params && !params_ok(*params)) return set_err(ctx, SHARP_EINVAL, "%s", "parameter out of range or not finite");
  const uint8_t *band = windows[rank] + SHARP_P2P_CTL_BYTES + (size_t)(in0 - (row0 - 4)) * w;
  if (!sharp::tma_supported(band, out, w, h))
    return set_err(ctx, SHARP_EUNSUPPORTED, "%s", "fused bands need the TMA path (8-byte aligned out)");
  sharp_params p;
  if (params) p = *params;
  else sharp_default_params(&p);
  const sharp::Params prm{p.amount, p.gamma, p.osc_gain, p.osc_scale};
  CK(cudaSetDevice(ctx->device));
  int rc;
  if ((rc = ensure_frames(ctx, 1))) return rc;
  CK(cudaMemsetAsync(ctx->zero_block, 0, ctx->zero_bytes, ctx->stream));
  sharp::BatchLaunch a;
  a.in = band;
  a.n = 1;
  a.out = out;
  a.acc = ctx->acc;
  a.sums = ctx->sums;
  a.means = ctx->means;
  a.luts = ctx->luts;
  a.lut_done = ctx->lut_done;
  a.task_counter = ctx->tcounters;
  const int set = (int)(epoch & 1) * 32;  // the partial slots' epoch-parity set (bands_p2p.cu)
  for (int g = 0; g < n_ranks; ++g) a.peer_slots[g] = reinterpret_cast<unsigned long long *>(windows[g]) + set + rank;
  a.my_slots = reinterpret_cast<const unsigned long long *>(windows[rank]) + set;
  a.epoch = epoch;
  a.ranks = n_ranks;
  a.grid_cap = grid_cap;
  if (halo) {  // the halo push of bands_p2p.cu inside the same launch
    auto ctl = [](uint8_t *win) { return reinterpret_cast<unsigned long long *>(win); };
    auto rows_of = [](uint8_t *win) { return win + SHARP_P2P_CTL_BYTES; };
    const int rows_own = row1 - row0;
    uint8_t *self = windows[rank];
    a.halo_on = 1;
    a.halo_bytes = 4 * w;
    a.self_ctl = ctl(self);
    a.own_top = rows_of(self) + (size_t)4 * w;
    a.own_bot = rows_of(self) + (size_t)rows_own * w;  // rows 4 + rows_own - 4 .. 4 + rows_own - 1
    if (rank > 0) {
      a.up_ctl = ctl(windows[rank - 1]);
      a.up_halo = rows_of(windows[rank - 1]) + (size_t)(4 + up_rows_own) * w;  // its lower halo
    }
    if (rank < n_ranks - 1) {
      a.down_ctl = ctl(windows[rank + 1]);
      a.down_halo = rows_of(windows[rank + 1]);  // its upper halo
    }
  }
  const double px = (double)(row1 - row0) * w;
  CK(timed(ctx, ctx->stream, 3, px, [&] {
    return sharp::launch_band_tma(a, sharp::kStepBandFused, w, h, row0, row1, in0, in1 - in0, prm, ctx->stream);
  }));
  ctx->last_frames = 1;
  ctx->stats.frames = 1;
  ctx->stats.kernels = 1;
  return SHARP_OK;
}

int sharp_band_p2p_allreduce(sharp_ctx *ctx, uint8_t *const *windows, int n_ranks, int rank,
                             const uint64_t *d_partial, uint64_t epoch, uint64_t *d_total) {
  NOT_MULTI(ctx);
  if (!ctx) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  if (!windows || !d_partial || !d_total || n_ranks < 1 || n_ranks > 32 || rank < 0 || rank >= n_ranks ||
      epoch == 0)
    return set_err(ctx, SHARP_EINVAL, "%s", "bad p2p all-reduce request (1 <= n_ranks <= 32, epoch > 0)");
  for (int g = 0; g < n_ranks; ++g)
    if (!windows[g] || ((uintptr_t)windows[g] & 15)) return set_err(ctx, SHARP_EINVAL, "%s", "bad window pointer");
  CK(sharp::launch_p2p_allreduce(windows, n_ranks, rank, reinterpret_cast<const unsigned long long *>(d_partial),
                                 epoch, reinterpret_cast<unsigned long long *>(d_total), ctx->stream));
  return SHARP_OK;
}

int sharp_ipc_get_handle(const void *d_ptr, void *handle) {
  if (!d_ptr || !handle) return SHARP_EINVAL;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, const_cast<void *>(d_ptr)) != cudaSuccess) {
    cudaGetLastError();
    return SHARP_ECUDA;
  }
  static_assert(sizeof(h) == SHARP_IPC_HANDLE_BYTES, "IPC handle size");
  memcpy(handle, &h, sizeof(h));
  return SHARP_OK;
}

int sharp_ipc_open_handle(const void *handle, void **d_ptr) {
  if (!handle || !d_ptr) return SHARP_EINVAL;
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  if (cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
    cudaGetLastError();
    *d_ptr = nullptr;
    return SHARP_ECUDA;
  }
  return SHARP_OK;
}

int sharp_ipc_close_handle(void *d_ptr) {
  if (!d_ptr) return SHARP_EINVAL;
  if (cudaIpcCloseMemHandle(d_ptr) != cudaSuccess) {
    cudaGetLastError();
    return SHARP_ECUDA;
  }
  return SHARP_OK;
}

int sharp_set_path(sharp_ctx *ctx, int path) {
  if (!ctx || path < SHARP_PATH_AUTO || path > SHARP_PATH_FUSED_EXP) return SHARP_EINVAL;
  if (ctx->poisoned) return SHARP_ESTATE;
  ctx->path = path;
  for (sharp_ctx *sc : ctx->sub) sc->path = path;  // multi-device: every device
  return SHARP_OK;
}

int sharp_get_path(const sharp_ctx *ctx) { return ctx ? ctx->path : SHARP_EINVAL; }

const char *sharp_strerror(int code) {
  switch (code) {
    case SHARP_OK: return "ok";
    case SHARP_EINVAL: return "invalid argument";
    case SHARP_ENOMEM: return "out of memory";
    case SHARP_ECUDA: return "CUDA error";
    case SHARP_ENCCL: return "communication error";
    case SHARP_EUNSUPPORTED: return "unsupported request";
    case SHARP_ESTATE: return "context poisoned by an earlier error";
    default: return "unknown error";
  }
}

const char *sharp_last_error(const sharp_ctx *ctx) { return ctx ? ctx->err : "no context"; }

const char *sharp_version(void) {
  return "libsharp 0.3 (sm_100a; persistent TMA step kernel, TMEM-resident kernel, two-pass, scalar fused and "
         "staged paths; general layouts; reading switches; multi-device contexts; peer-memory row bands)";
}

}  // extern "C"
