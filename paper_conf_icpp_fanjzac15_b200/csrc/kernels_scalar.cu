// Scalar fused kernels: the "+fusion" rungs of the optimisation ladder
// (sec. V-B; Fig. 14), between the paper's
// staged base design (kernels_staged.cu: every stage a kernel, every matrix in
// HBM) and the vectorised two-pass kernels (kernels.cu).  One thread per
// pixel, no SIMD pairs, no data reuse between pixels (each thread loads its
// own 3x3 window and D values: the "8 loads per pixel" of L342-L346), but the
// stages are fused:
//   K1  downscale O -> D (f32, 1/16 of the pixels; the paper's fused kernel
//       also read the downscaled matrix from global memory)
//   P1  Sobel + block reduction + one u64 atomic per warp (L158-L174)
//   [T  per-frame table {adj, osc}(pEdge) from the mean, f64 rounded once]
//   P2  upscale (body L146 from D, border L140-L142), pError, Sobel again,
//       3x3 max/min, strength, preliminary, overshoot, RNE -> u8
// Two variants of P2: strength and oscStrength evaluated per pixel in f64
// (the paper's fused kernel: "many exponentiations", L232) or looked up in
// the per-frame table.  Same arithmetic as every other path (R15):
// bit-identical outputs.
#include <cuda_runtime.h>
#include <stdint.h>

#include "device_common.cuh"
#include "kernels.h"

namespace sharp {
namespace {
using namespace dev;

constexpr int kBX = 32, kBY = 8;  // 256 threads, one pixel each

__global__ void sc_downscale(const uint8_t *__restrict__ O, int W, int w, int h, float *__restrict__ D) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x, i = blockIdx.y;
  if (j >= w || i >= h) return;
  unsigned s = 0;
#pragma unroll
  for (int a = 0; a < 4; ++a)
#pragma unroll
    for (int b = 0; b < 4; ++b) s += O[(size_t)(4 * i + a) * W + 4 * j + b];
  D[(size_t)i * w + j] = __fmul_rn((float)s, 1.0f / 16.0f);  // L130, exact (R2)
}

__device__ __forceinline__ int sobel_at(const uint8_t *__restrict__ O, int W, int H, int r, int c) {
  if (r <= 0 || c <= 0 || r >= H - 1 || c >= W - 1) return 0;  // L160: the frame is 0
  auto o = [&](int rr, int cc) { return (int)__ldg(O + (size_t)rr * W + cc); };
  const int gx = (o(r - 1, c + 1) + 2 * o(r, c + 1) + o(r + 1, c + 1)) - (o(r - 1, c - 1) + 2 * o(r, c - 1) + o(r + 1, c - 1));
  const int gy = (o(r + 1, c - 1) + 2 * o(r + 1, c) + o(r + 1, c + 1)) - (o(r - 1, c - 1) + 2 * o(r - 1, c) + o(r - 1, c + 1));
  return abs(gx) + abs(gy);  // L166, R7
}

__global__ void sc_edge_sum(const uint8_t *__restrict__ O, int W, int H, unsigned long long *sum) {
  const int c = blockIdx.x * kBX + threadIdx.x, r = blockIdx.y * kBY + threadIdx.y;
  const int pe = (c < W && r < H) ? sobel_at(O, W, H, r, c) : 0;
  const unsigned ws = __reduce_add_sync(0xffffffffu, (unsigned)pe);  // L174: one atomic per warp
  if ((threadIdx.x & 31) == 0 && ws) atomicAdd(sum, (unsigned long long)ws);
}

__global__ void sc_table(const unsigned long long *sum, int W, int H, Params prm, double *mean_out,
                         float2 *__restrict__ lut) {
  const double mean = frame_mean(*sum, W, H, prm.flags);
  if (threadIdx.x == 0) *mean_out = mean;
  for (int p = threadIdx.x; p <= 1530; p += blockDim.x) lut[p] = lut_entry(p, mean, prm);
}

// U at (r, c) from D (R3-R5): body bilinear, 2-pixel ring by the step rules.
__device__ __forceinline__ float u_at(const float *__restrict__ D, int w, int h, int W, int H, int r, int c) {
  const int c0 = c & ~7, x = c - c0, j0 = c0 >> 2, k = r >> 2;
  auto S = [&](int i, int j) {  // 16 * D[i][j] (exact), 0 outside (unused there)
    return (i >= 0 && i < h && j >= 0 && j < w) ? __fmul_rn(__ldg(D + (size_t)i * w + j), 16.0f) : 0.0f;
  };
  if (r < 2 || r >= H - 2 || c < 2 || c >= W - 2) {
    float Sc[4], Sn[4];
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      Sc[t] = S(k, j0 - 1 + t);
      Sn[t] = S(k + 1, j0 - 1 + t);
    }
    return ring_u(r, c, W, H, j0, Sc, Sn, false);
  }
  const int a = r & 3;
  const float wt = (float)(a == 0 ? 3 : a == 1 ? 1 : a == 2 ? 7 : 5), wb = 8.0f - wt;
  const int it = a < 2 ? k - 1 : k, jl = j0 - 1 + jl_of(x);
  const float wl = (float)wl_of(x);
  const float Vl = __fmaf_rn(wb, S(it + 1, jl), __fmul_rn(wt, S(it, jl)));
  const float Vr = __fmaf_rn(wb, S(it + 1, jl + 1), __fmul_rn(wt, S(it, jl + 1)));
  return -__fmaf_rn(-(8.0f - wl) * (1.0f / 1024.0f), Vr, __fmul_rn(-wl * (1.0f / 1024.0f), Vl));
}

template <bool kTable>
__global__ void sc_sharpen(const uint8_t *__restrict__ O, const float *__restrict__ D, int W, int H, Params prm,
                           const double *mean_in, const float2 *__restrict__ lut, uint8_t *__restrict__ out) {
  const int c = blockIdx.x * kBX + threadIdx.x, r = blockIdx.y * kBY + threadIdx.y;
  if (c >= W || r >= H) return;
  const int w = W >> 2, h = H >> 2;
  const float U = u_at(D, w, h, W, H, r, c);
  const int o = __ldg(O + (size_t)r * W + c);
  const float E = __fsub_rn((float)o, U);  // L148 (exact)
  const int pe = sobel_at(O, W, H, r, c);
  float mxf = 255.0f, mnf = 0.0f;  // frame: the clamped preliminary value (R13)
  if (r > 0 && c > 0 && r < H - 1 && c < W - 1) {
    int mx = 0, mn = 255;
#pragma unroll
    for (int a = -1; a <= 1; ++a)
#pragma unroll
      for (int b = -1; b <= 1; ++b) {
        const int v = __ldg(O + (size_t)(r + a) * W + c + b);
        mx = max(mx, v);
        mn = min(mn, v);
      }
    mxf = (float)mx;
    mnf = (float)mn;
  }
  float2 L;
  if (kTable) L = lut[pe];
  else L = lut_entry(pe, *mean_in, prm);  // per-pixel f64 exponentiation (L232)
  out[(size_t)r * W + c] = (uint8_t)sharpen_px(L.x, L.y, E, U, mxf, mnf);
}

}  // namespace

static size_t d_bytes(int W, int H) { return ((size_t)(W / 4) * (H / 4) * sizeof(float) + 255) & ~(size_t)255; }

size_t scalar_scratch_bytes(int W, int H) { return d_bytes(W, H) + (size_t)kLutSize * sizeof(float2); }

cudaError_t launch_scalar(const uint8_t *in, int W, int H, const Params &p, void *scratch, unsigned long long *sum,
                          double *mean, uint8_t *out, bool table, cudaStream_t st) {
  const int w = W / 4, h = H / 4;
  float *D = static_cast<float *>(scratch);
  float2 *lut = reinterpret_cast<float2 *>(static_cast<uint8_t *>(scratch) + d_bytes(W, H));  // 256-B aligned
  sc_downscale<<<dim3((w + 127) / 128, h), 128, 0, st>>>(in, W, w, h, D);
  const dim3 grid((W + kBX - 1) / kBX, (H + kBY - 1) / kBY), block(kBX, kBY);
  sc_edge_sum<<<grid, block, 0, st>>>(in, W, H, sum);
  sc_table<<<1, 768, 0, st>>>(sum, W, H, p, mean, lut);  // mean (and the table, used when `table`)
  if (table) sc_sharpen<true><<<grid, block, 0, st>>>(in, D, W, H, p, mean, lut, out);
  else sc_sharpen<false><<<grid, block, 0, st>>>(in, D, W, H, p, mean, lut, out);
  return cudaGetLastError();
}

cudaError_t preload_scalar() {
  cudaFuncAttributes a;
  cudaError_t e;
  if ((e = cudaFuncGetAttributes(&a, sc_downscale)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, sc_edge_sum)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, sc_table)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, sc_sharpen<true>)) != cudaSuccess) return e;
  return cudaFuncGetAttributes(&a, sc_sharpen<false>);
}

}  // namespace sharp
