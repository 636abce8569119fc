// Internal launch interface of the sm_100a kernels (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace sharp {

// Lookup tables built once per frame by the last CTA of pass 1: entry p
// (p = pEdge value, 0..1530 = 6*255) holds {adj(p), osc(p)} (R9, R11).
constexpr int kLutSize = 1536;

struct Params {
  float amount, gamma, osc_gain, osc_scale;
};

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
                           uint8_t *outs, cudaStream_t stream);

// TMA-staged, dynamically scheduled step kernel (kernels_tma.cu), used when
// tma_supported() (W % 16 == 0, 16-byte aligned input, 8-byte aligned output).
// One launch = LUT build (mean from the complete sums) + pass 2 of chunk "2"
// (n2 frames, may be 0) and pass 1 of chunk "1" (n1 frames, may be 0).
// Chunk 2's sums must be complete (an earlier launch's pass 1); chunk 1's
// sums, lut_done2 and task_counter must be zero on entry.
struct StepLaunch {
  const uint8_t *in1 = nullptr;
  int n1 = 0;
  unsigned long long *sums1 = nullptr;
  const uint8_t *in2 = nullptr;
  int n2 = 0;
  const unsigned long long *sums2 = nullptr;
  double *means2 = nullptr;
  float2 *luts2 = nullptr;
  unsigned int *lut_done2 = nullptr;
  uint8_t *out2 = nullptr;
  unsigned int *task_counter = nullptr;
};
bool tma_supported(const uint8_t *imgs, const uint8_t *outs, int W, int H);
cudaError_t launch_step_tma(const StepLaunch &a, int W, int H, const Params &p, cudaStream_t stream);

// Kernel launches issued per (pass-1, pass-2) chunk.
constexpr int kLaunchesPerChunk = 2;

}  // namespace sharp
