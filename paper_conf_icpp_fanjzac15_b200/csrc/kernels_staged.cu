// The paper's BASE GPU design (sec. IV; Fig. 13(b) stage list):
// one plain kernel per stage of sec. III, every intermediate matrix
// materialised in HBM, one thread per element.  It is the first rung of the
// optimisation ladder (SHARP_PATH_STAGED) that the fused kernels are
// measured against (Fig. 12 / Fig. 14),
// and it gives the per-stage time breakdown (Fig. 13).  Same arithmetic and
// readings as the fused kernels, so bit-identical output.
//
//   K1 downscale      O (u8)        -> D  (f32, h x w)          L130, L136
//   K2 border         D             -> U ring (f32, H x W)      L138-L142 (steps i-vii)
//   K3 center         D             -> U body                   L146 (R3)
//   K4 sobel          O             -> pE (u16, H x W)          L158-L172 (R7)
//   K5 reduction      pE            -> S (u64)                  L174, sec. V-C
//   K6 strength       pE, S         -> {adj, osc} (f32x2/px)    L178, L184, L232 (R9, R11)
//   K7 sharpness      O, U, adj/osc -> out (u8)                 L178-L212, Fig. 8
#include <cuda_runtime.h>
#include <stdint.h>

#include "device_common.cuh"
#include "kernels.h"

namespace sharp {
namespace {

// ---------------------------------------------------------------- K1
__global__ void st_downscale(const uint8_t *__restrict__ O, int W, int h, int w, int flags, float *__restrict__ D) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x, i = blockIdx.y;
  if (j >= w || i >= h) return;
  unsigned s = 0;
  for (int a = 0; a < 4; ++a) {
    const uint32_t v = *reinterpret_cast<const uint32_t *>(O + (size_t)(4 * i + a) * W + 4 * j);
    s += (v & 0xff) + ((v >> 8) & 0xff) + ((v >> 16) & 0xff) + (v >> 24);
  }
  // mean of the 4x4 block (R2, exact), or the integer shift s >> 4 (the R2 alternative, L374)
  D[(size_t)i * w + j] = (flags & kReadIntDownscale) ? (float)(s >> 4) : __fmul_rn((float)s, 1.0f / 16.0f);
}

// ---------------------------------------------------------------- K2
// lerp_k(x, y) = ((4-k) x + k y) / 4 (exact in f32 for x, y multiples of 1/16 <= 255)
__device__ __forceinline__ float lerp4(float x, float y, int k) {
  return __fmul_rn(__fadd_rn(__fmul_rn((float)(4 - k), x), __fmul_rn((float)k, y)), 0.25f);
}
// line(v, n)[c] for c in [0, n-3] (L140): D every fourth element, the
// vacancies interpolated, the third-last element copied from the fourth-last.
__device__ __forceinline__ float line_at(const float *v, size_t stride, int n, int c) {
  if (c == n - 3) c = n - 4;
  const int j = c >> 2, k = c & 3;
  return k == 0 ? v[(size_t)j * stride] : lerp4(v[(size_t)j * stride], v[(size_t)(j + 1) * stride], k);
}
// One CTA walks the steps (i)..(vii) of L140-L142 in order (the border is
// 4(W+H) elements; __syncthreads orders the overlapping steps).  With the R5
// alternative the row copies (v) run before the column lines (ii), (iv).
__global__ void st_border(const float *__restrict__ D, int W, int H, int w, int h, int flags,
                          float *__restrict__ U) {
  const int t = threadIdx.x, nt = blockDim.x;
  const bool col_wins = (flags & kReadColumnWins) != 0;
  // (i) row 0 and (iii) row H-2: lines of D rows 0 and h-1 over columns 0..W-3
  for (int c = t; c <= W - 3; c += nt) {
    U[c] = line_at(D, 1, W, c);
    U[(size_t)(H - 2) * W + c] = line_at(D + (size_t)(h - 1) * w, 1, W, c);
  }
  __syncthreads();
  for (int pass = 0; pass < 2; ++pass) {
    if ((pass == 0) != col_wins) {
      // (ii) column 0 and (iv) column W-2: lines of D columns 0 and w-1 over rows 0..H-3
      for (int r = t; r <= H - 3; r += nt) {
        U[(size_t)r * W] = line_at(D, (size_t)w, H, r);
        U[(size_t)r * W + W - 2] = line_at(D + (w - 1), (size_t)w, H, r);
      }
    } else {
      // (v) copy row 0 -> 1 and row H-2 -> H-1 over columns 0..W-3
      for (int c = t; c <= W - 3; c += nt) {
        U[(size_t)W + c] = U[c];
        U[(size_t)(H - 1) * W + c] = U[(size_t)(H - 2) * W + c];
      }
    }
    __syncthreads();
  }
  // (vi) copy column 0 -> 1 and column W-2 -> W-1 over rows 0..H-3
  for (int r = t; r <= H - 3; r += nt) {
    U[(size_t)r * W + 1] = U[(size_t)r * W];
    U[(size_t)r * W + W - 1] = U[(size_t)r * W + W - 2];
  }
  __syncthreads();
  // (vii) the four bottom-right elements (L142) <- U[H-3][W-1]
  if (t == 0) {
    const float v = U[(size_t)(H - 3) * W + W - 1];
    U[(size_t)(H - 2) * W + W - 2] = v;
    U[(size_t)(H - 2) * W + W - 1] = v;
    U[(size_t)(H - 1) * W + W - 2] = v;
    U[(size_t)(H - 1) * W + W - 1] = v;
  }
}

// ---------------------------------------------------------------- K3
// U[4i+2+a][4j+2+b] = sum_{p,q} P[a][p] P[b][q] D[i+p][j+q],
// P = [[7,1],[5,3],[3,5],[1,7]] / 8 (R3); every partial result is exact.
__global__ void st_center(const float *__restrict__ D, int W, int H, int w, float *__restrict__ U) {
  const int c = 2 + blockIdx.x * blockDim.x + threadIdx.x, r = 2 + blockIdx.y;
  if (c > W - 3 || r > H - 3) return;
  const int i = (r - 2) >> 2, a = (r - 2) & 3, j = (c - 2) >> 2, b = (c - 2) & 3;
  const float pa0 = (float)(7 - 2 * a), pa1 = (float)(1 + 2 * a);
  const float pb0 = (float)(7 - 2 * b), pb1 = (float)(1 + 2 * b);
  const float *d0 = D + (size_t)i * w + j, *d1 = d0 + w;
  const float top = __fadd_rn(__fmul_rn(pb0, d0[0]), __fmul_rn(pb1, d0[1]));
  const float bot = __fadd_rn(__fmul_rn(pb0, d1[0]), __fmul_rn(pb1, d1[1]));
  U[(size_t)r * W + c] = __fmul_rn(__fadd_rn(__fmul_rn(pa0, top), __fmul_rn(pa1, bot)), 1.0f / 64.0f);
}

// ---------------------------------------------------------------- K4
__global__ void st_sobel(const uint8_t *__restrict__ O, int W, int H, uint16_t *__restrict__ pE) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x, r = blockIdx.y;
  if (c >= W || r >= H) return;
  int v = 0;
  if (r > 0 && r < H - 1 && c > 0 && c < W - 1) {  // the frame is 0 (L160)
    const uint8_t *a = O + (size_t)(r - 1) * W + c, *b = a + W, *d = b + W;
    const int gx = (a[1] + 2 * b[1] + d[1]) - (a[-1] + 2 * b[-1] + d[-1]);
    const int gy = (d[-1] + 2 * d[0] + d[1]) - (a[-1] + 2 * a[0] + a[1]);
    v = abs(gx) + abs(gy);
  }
  pE[(size_t)r * W + c] = (uint16_t)v;
}

// ---------------------------------------------------------------- K5
// Two-level reduction (sec. V-C): block tree in shared memory, one u64
// atomic per block.
__global__ void st_reduce(const uint16_t *__restrict__ pE, size_t n, unsigned long long *S) {
  __shared__ unsigned int part[256];
  unsigned int s = 0;
  for (size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x; k < n; k += (size_t)gridDim.x * blockDim.x)
    s += pE[k];
  part[threadIdx.x] = s;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if ((int)threadIdx.x < o) part[threadIdx.x] += part[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) atomicAdd(S, (unsigned long long)part[0]);
}

// ---------------------------------------------------------------- K6
// Per-pixel brightness strength (the "many exponentiations" of L232):
// adj = A (p / m)^gamma, osc = clamp(G exp(-p / (K m)), 0, 1), f64 rounded
// once to f32 (R9, R11, R15); thread (0,0) also stores the mean (L174, R8).
__global__ void st_strength(const uint16_t *__restrict__ pE, size_t n, const unsigned long long *S, int W, int H,
                            Params prm, float2 *__restrict__ ao, double *mean_out) {
  const double mean = dev::frame_mean(*S, W, H, prm.flags);
  const size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  if (k == 0) *mean_out = mean;
  if (k >= n) return;
  ao[k] = dev::lut_entry(pE[k], mean, prm);
}

// ---------------------------------------------------------------- K7
// pError E = O - U (L148, R6), preliminary P = fma(adj, E, U) (L178, R10),
// overshoot control of Fig. 8 (L180-L212, R11-R13), RNE to 8 bits (R14).
__global__ void st_sharpen(const uint8_t *__restrict__ O, const float *__restrict__ U,
                           const float2 *__restrict__ ao, int W, int H, int flags, uint8_t *__restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x, r = blockIdx.y;
  if (c >= W || r >= H) return;
  const size_t k = (size_t)r * W + c;
  const float u = U[k];
  const float2 s = ao[k];
  const float E = __fsub_rn((float)O[k], u);
  const float P = __fmaf_rn(s.x, E, u);
  float F;
  if (r == 0 || r == H - 1 || c == 0 || c == W - 1) {
    F = fminf(fmaxf(P, 0.0f), 255.0f);  // the frame copies the preliminary value (L208, R13)
  } else {
    int mx = 0, mn = 255;
    for (int dr = -1; dr <= 1; ++dr)
      for (int dc = -1; dc <= 1; ++dc) {
        const int v = O[k + (ptrdiff_t)dr * W + dc];
        mx = max(mx, v);
        mn = min(mn, v);
      }
    const float mxf = (float)mx, mnf = (float)mn;
    if (P > mxf) F = fminf(__fmaf_rn(s.y, __fsub_rn(P, mxf), mxf), 255.0f);       // osc max
    else if (P < mnf) F = fmaxf(__fmaf_rn(s.y, __fsub_rn(P, mnf), mnf), 0.0f);   // osc min
    else F = fminf(fmaxf(P, 0.0f), 255.0f);
  }
  out[k] = (uint8_t)((flags & kReadTruncate) ? __float2int_rz(F) : __float2int_rn(F));  // R14
}

}  // namespace

size_t staged_scratch_bytes(int W, int H) {
  const size_t px = (size_t)W * H, d = (size_t)(W / 4) * (H / 4);
  return d * 4 + px * 4 + px * 2 + px * 8 + 256 * 5;
}

cudaError_t launch_staged(const uint8_t *in, int W, int H, const Params &p, void *scratch,
                          unsigned long long *sum, double *mean, uint8_t *out, cudaStream_t st,
                          const StageTimer &timer) {
  const int w = W / 4, h = H / 4;
  const size_t px = (size_t)W * H;
  uint8_t *base = static_cast<uint8_t *>(scratch);
  auto align = [](size_t x) { return (x + 255) & ~(size_t)255; };
  float *D = reinterpret_cast<float *>(base);
  float *U = reinterpret_cast<float *>(base + align((size_t)w * h * 4));
  uint16_t *pE = reinterpret_cast<uint16_t *>(reinterpret_cast<uint8_t *>(U) + align(px * 4));
  float2 *ao = reinterpret_cast<float2 *>(reinterpret_cast<uint8_t *>(pE) + align(px * 2));
  const int tb = 256;
  cudaError_t e;
  timer.begin(kStageDownscale, st);
  st_downscale<<<dim3((w + tb - 1) / tb, h), tb, 0, st>>>(in, W, h, w, p.flags, D);
  timer.end(kStageDownscale, st);
  timer.begin(kStageBorder, st);
  st_border<<<1, 1024, 0, st>>>(D, W, H, w, h, p.flags, U);
  timer.end(kStageBorder, st);
  timer.begin(kStageCenter, st);
  st_center<<<dim3((W - 4 + tb - 1) / tb, H - 4), tb, 0, st>>>(D, W, H, w, U);
  timer.end(kStageCenter, st);
  timer.begin(kStageSobel, st);
  st_sobel<<<dim3((W + tb - 1) / tb, H), tb, 0, st>>>(in, W, H, pE);
  timer.end(kStageSobel, st);
  timer.begin(kStageReduce, st);
  if ((e = cudaMemsetAsync(sum, 0, sizeof(*sum), st)) != cudaSuccess) return e;
  st_reduce<<<148 * 8, 256, 0, st>>>(pE, px, sum);
  timer.end(kStageReduce, st);
  timer.begin(kStageStrength, st);
  st_strength<<<(unsigned)((px + tb - 1) / tb), tb, 0, st>>>(pE, px, sum, W, H, p, ao, mean);
  timer.end(kStageStrength, st);
  timer.begin(kStageSharpen, st);
  st_sharpen<<<dim3((W + tb - 1) / tb, H), tb, 0, st>>>(in, U, ao, W, H, p.flags, out);
  timer.end(kStageSharpen, st);
  return cudaGetLastError();
}

// Forces the (lazy) module load of this file's kernels; see kernels.h.
cudaError_t preload_staged() {
  cudaFuncAttributes a;
  cudaError_t e;
  if ((e = cudaFuncGetAttributes(&a, st_downscale)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, st_border)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, st_center)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, st_sobel)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, st_reduce)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, st_strength)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, st_sharpen)) != cudaSuccess) return e;
  return cudaSuccess;
}

}  // namespace sharp
