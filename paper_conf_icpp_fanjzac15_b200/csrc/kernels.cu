// sm_100a kernels of the sharpness pipeline (sec. III).
//
// Two passes per chunk of frames (the pEdge mean, L174, is a global
// dependency of every output pixel):
//   pass 1  edge_sum_kernel : Sobel (L158-L172) + reduction (L174, sec. V-C)
//           -> per-CTA u32 partial via warp reductions -> u64 atomic -> the
//           last CTA of a frame computes the mean and both per-frame lookup
//           tables (strength L178 / oscStrength L184), "last-block-done".
//   pass 2  sharpen_kernel  : downscale (L130) + upscale body/border
//           (L140-L146) + pError (L148) + Sobel + 3x3 max/min (L182) +
//           strength lookup + preliminary (L178) + overshoot (L180-L212)
//           -> u8, all in registers (the paper's "sharpness" fusion, L280,
//           extended to every stage).
// Chunks are sized so a chunk's input stays in L2 between the passes, so HBM
// sees ~1 B/px in + 1 B/px out.
//
// Work decomposition: a warp owns a 256-column x 32-row tile; each lane owns
// 8 adjacent columns (two 32-bit words per row) and walks down the rows with a
// 3-row sliding window in registers.  Pixels are held as f16x2 pairs (even /
// odd columns of each word) so the Sobel / max / min arithmetic runs two
// pixels per instruction; all of it is exact (integers < 2048).  Halo
// columns come from the neighbouring lanes by shuffle.
//
// Arithmetic (R15): D, U and pError are exact (dyadic rationals);
// P = fma(adj, E, U) and the overshoot fma are single-rounding f32, exactly
// as the oracle; the lookup tables are evaluated in f64 and rounded once.
#include <cuda_fp16.h>
#include <stdint.h>

#include "device_common.cuh"
#include "kernels.h"

namespace sharp {
namespace {

constexpr int kPx = 8;                 // pixels per lane per row
constexpr int kWarpCols = 32 * kPx;    // 256 columns per warp tile
constexpr int kTileRows = 32;          // rows per warp tile (multiple of 4)
constexpr int kWarps = 4;              // warps per CTA
constexpr int kThreads = kWarps * 32;
constexpr int kLutEven = 766;          // entries k = pEdge / 2, pEdge in [0, 1530]

using namespace dev;

__device__ __forceinline__ uint32_t ldw(const uint8_t *__restrict__ img, int W, int H, int r, int c) {
  if (r < 0 || r >= H || c < 0 || c >= W) return 0u;  // outside the image: 0
  return __ldg(reinterpret_cast<const uint32_t *>(img + (size_t)r * W + c));
}

// All 32 lanes must call this (shuffles).
__device__ __forceinline__ Words load_row(const uint8_t *__restrict__ img, int W, int H, int r, int c0,
                                          int lane) {
  Words x;
  x.w0 = ldw(img, W, H, r, c0);
  x.w1 = ldw(img, W, H, r, c0 + 4);
  x.pw = __shfl_up_sync(0xffffffffu, x.w1, 1);
  x.nw = __shfl_down_sync(0xffffffffu, x.w0, 1);
  if (lane == 0) x.pw = ldw(img, W, H, r, c0 - 4);
  if (lane == 31) x.nw = ldw(img, W, H, r, c0 + 8);
  return x;
}

struct Block {  // 4 rows of words + the four D sums (16*D) of columns j0-1..j0+2
  Words r[4];
  float S[4];
};

// S = 16 * D; with the R2 alternative (integer downscale) D = floor(sum / 16),
// i.e. S = sum with its low 4 bits cleared.
__device__ __forceinline__ void load_block(Block &B, const uint8_t *__restrict__ img, int W, int H, int k,
                                           int c0, int lane, uint32_t smask) {
#pragma unroll
  for (int a = 0; a < 4; ++a) B.r[a] = load_row(img, W, H, 4 * k + a, c0, lane);
  B.S[0] = (float)(blk4(B.r[0].pw, B.r[1].pw, B.r[2].pw, B.r[3].pw) & smask);
  B.S[1] = (float)(blk4(B.r[0].w0, B.r[1].w0, B.r[2].w0, B.r[3].w0) & smask);
  B.S[2] = (float)(blk4(B.r[0].w1, B.r[1].w1, B.r[2].w1, B.r[3].w1) & smask);
  B.S[3] = (float)(blk4(B.r[0].nw, B.r[1].nw, B.r[2].nw, B.r[3].nw) & smask);
}

// =========================================================================
// Pass 1: Sobel + reduction + last-block-done LUT construction.
// =========================================================================
__global__ void __launch_bounds__(kThreads) edge_sum_kernel(const uint8_t *__restrict__ imgs, int W, int H,
                                                            int tiles_x, int tiles_y, Params prm,
                                                            unsigned long long *__restrict__ sums,
                                                            unsigned int *__restrict__ counters,
                                                            float2 *__restrict__ luts,
                                                            double *__restrict__ means) {
  __shared__ uint32_t warp_sum[kWarps];
  __shared__ int am_last;
  const int f = blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int tile = blockIdx.x * kWarps + warp;
  const uint8_t *img = imgs + (size_t)f * W * H;
  float acc = 0.0f;  // exact: < 8 px * 32 rows * 1530 < 2^24
  if (tile < tiles_x * tiles_y) {
    const int tx = tile % tiles_x, ty = tile / tiles_x;
    const int c0 = tx * kWarpCols + lane * kPx;
    const int R0 = ty * kTileRows;
    const int R1 = min(R0 + kTileRows, H);
    RowD a = derive<false>(load_row(img, W, H, R0 - 1, c0, lane));
    RowD b = derive<false>(load_row(img, W, H, R0, c0, lane));
    for (int r = R0; r < R1; ++r) {
      const RowD c = derive<false>(load_row(img, W, H, r + 1, c0, lane));
      uint32_t pe[4];
      sobel(a, b, c, pe);
      if (r == 0 || r == H - 1) {  // Sobel border rows are 0 (L160)
#pragma unroll
        for (int i = 0; i < 4; ++i) pe[i] = 0u;
      }
      if (c0 == 0) set_px(pe, 0, 0u);                          // first column
      if (c0 <= W - 1 && W - 1 < c0 + kPx) set_px(pe, W - 1 - c0, 0u);  // last column
      if (c0 + kPx > W) {                                       // pixels beyond the image
#pragma unroll
        for (int x = 0; x < kPx; ++x)
          if (c0 + x >= W) set_px(pe, x, 0u);
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        acc = add_f32_f16(lo16(pe[i]), acc);
        acc = add_f32_f16(hi16(pe[i]), acc);
      }
      a = b;
      b = c;
    }
  }
  // Reduction stage 1 (sec. V-C, Fig. 9): warp reduction then CTA partial.
  const uint32_t ws = __reduce_add_sync(0xffffffffu, (uint32_t)acc);
  if (lane == 0) warp_sum[warp] = ws;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long part = 0;
#pragma unroll
    for (int i = 0; i < kWarps; ++i) part += warp_sum[i];
    atomicAdd(&sums[f], part);
    __threadfence();
    const unsigned int ticket = atomicAdd(&counters[f], 1u);
    am_last = (ticket == gridDim.x - 1);
  }
  __syncthreads();
  if (!am_last) return;
  // Stage 2 (last-block-done): mean and the per-frame lookup tables.
  __threadfence();
  const unsigned long long S = atomicAdd(&sums[f], 0ull);
  const double mean = frame_mean(S, W, H, prm.flags);
  // even pEdge values only (pEdge is always even: Gx and Gy have the parity
  // of the sum of the window's corners): entry k = lut(2k), k < kLutEven
  for (int k = threadIdx.x; k < kLutEven; k += kThreads)
    luts[(size_t)f * kLutSize + k] = lut_entry(2 * k, mean, prm);
  if (threadIdx.x == 0) {
    means[f] = mean;
    counters[f] = 0u;  // re-arm for the next launch
  }
}

// =========================================================================
// Pass 2: everything else, fused.
// =========================================================================
__global__ void __launch_bounds__(kThreads) sharpen_kernel(const uint8_t *__restrict__ imgs, int W, int H,
                                                           int tiles_x, int tiles_y,
                                                           const float2 *__restrict__ luts,
                                                           uint8_t *__restrict__ outs, int flags) {
  __shared__ float2 lut[kLutEven];
  const int f = blockIdx.y;
  for (int i = threadIdx.x; i < kLutEven; i += kThreads) lut[i] = luts[(size_t)f * kLutSize + i];
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int tile = blockIdx.x * kWarps + warp;
  if (tile >= tiles_x * tiles_y) return;
  // LDS address of lut[p] from the bits of (2^23 + p) as f32: q*8 + base'.
  // byte offset of entry k = pEdge/2: the f32 bits of 2^21 + pEdge minus
  // 0x4A000000 (ulp 1/4, so 8k); the shared base is uniform (LDS [R+UR])
  // (the vote makes the base provably warp-uniform: ptxas keeps it in a uniform register)
  const uint32_t lut_base =
      (__any_sync(0xffffffffu, (threadIdx.x & 31) == 0) ? (uint32_t)__cvta_generic_to_shared(lut) : 0u) - 0x4A000000u;

  const int tx = tile % tiles_x, ty = tile / tiles_x;
  const int c0 = tx * kWarpCols + lane * kPx;
  const int j0 = c0 >> 2;
  const int R0 = ty * kTileRows;  // multiple of 4
  const int R1 = min(R0 + kTileRows, H);
  const uint8_t *img = imgs + (size_t)f * W * H;
  uint8_t *out = outs + (size_t)f * W * H;
  const bool ring_cols = (c0 < 2) || (c0 + kPx > W - 2);

  const uint32_t smask = (flags & kReadIntDownscale) ? ~15u : ~0u;
  const bool col_wins = (flags & kReadColumnWins) != 0, trunc = (flags & kReadTruncate) != 0;
  Block prev, cur, next;
  load_block(prev, img, W, H, (R0 >> 2) - 1, c0, lane, smask);
  load_block(cur, img, W, H, R0 >> 2, c0, lane, smask);
  RowD ra = derive<true>(prev.r[3]);
  RowD rb = derive<true>(cur.r[0]);

  for (int k = R0 >> 2; 4 * k < R1; ++k) {
    load_block(next, img, W, H, k + 1, c0, lane, smask);
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      const int r = 4 * k + a;
      const RowD rc = derive<true>(a < 3 ? cur.r[a + 1] : next.r[0]);
      if (r < R1) {
        uint32_t pe[4], MX[4], MN[4];
        sobel(ra, rb, rc, pe);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          MX[i] = __vimax3_u16x2(ra.mx[i], rb.mx[i], rc.mx[i]);
          MN[i] = __vimin3_u16x2(ra.mn[i], rb.mn[i], rc.mn[i]);
        }
        // Frame of the image: Sobel 0 (L160) and no overshoot window (L208,
        // R13: the frame is the clamped preliminary value == window [0,255]).
        if (r == 0 || r == H - 1) {
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            pe[i] = 0u;
            MX[i] = kF16_255 | (kF16_255 << 16);
            MN[i] = 0u;
          }
        }
        if (c0 == 0) {
          set_px(pe, 0, 0u);
          set_px(MX, 0, kF16_255);
          set_px(MN, 0, 0u);
        }
        if (c0 <= W - 1 && W - 1 < c0 + kPx) {
          set_px(pe, W - 1 - c0, 0u);
          set_px(MX, W - 1 - c0, kF16_255);
          set_px(MN, W - 1 - c0, 0u);
        }
        // Vertical interpolation of the three D-column sums (16*D):
        //   a' = 0,1: U block row k-1, weights (3,5),(1,7) on D rows (k-1,k)
        //   a' = 2,3: U block row k,   weights (7,1),(5,3) on D rows (k,k+1)
        const float wt = (float)(a == 0 ? 3 : a == 1 ? 1 : a == 2 ? 7 : 5);
        const float wb = 8.0f - wt;
        float V[4];  // 128 * D interpolated vertically (exact)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float top = a < 2 ? prev.S[j] : cur.S[j];
          const float bot = a < 2 ? cur.S[j] : next.S[j];
          V[j] = __fmaf_rn(wb, bot, __fmul_rn(wt, top));
        }
        float NU[8];  // -U, exact
#pragma unroll
        for (int x = 0; x < 8; ++x) {
          const int jl = jl_of(x);
          const float wl = (float)wl_of(x);
          NU[x] = __fmaf_rn(-(8.0f - wl) * (1.0f / 1024.0f), V[jl + 1], __fmul_rn(-wl * (1.0f / 1024.0f), V[jl]));
        }
        if (r < 2 || r >= H - 2 || ring_cols) {  // the 2-pixel upscale border ring
          const float(&Sc)[4] = cur.S;  // D row k: row 0 for rows 0,1; row h-1 for rows H-2,H-1
          const float(&Sn)[4] = next.S;
#pragma unroll
          for (int x = 0; x < 8; ++x) {
            const int c = c0 + x;
            if (c < W && (r < 2 || r >= H - 2 || c < 2 || c >= W - 2)) NU[x] = -ring_u(r, c, W, H, j0, Sc, Sn, col_wins);
          }
        }
        float F8[8];
#pragma unroll
        for (int x = 0; x < 8; ++x) {
          const int p = pair_of(x);
          const bool hi = half_of(x);
          const uint16_t pe_h = hi ? hi16(pe[p]) : lo16(pe[p]);
          const uint16_t c_h = hi ? hi16(rb.c[p]) : lo16(rb.c[p]);
          const uint16_t mx_h = hi ? hi16(MX[p]) : lo16(MX[p]);
          const uint16_t mn_h = hi ? hi16(MN[p]) : lo16(MN[p]);
          const uint32_t q8 = __float_as_uint(add_f32_f16(pe_h, 2097152.0f));  // 2^21 + pEdge
          const float2 L = lds_f2(q8 + lut_base);                               // {adj, osc}
          const float E = add_f32_f16(c_h, NU[x]);                           // pError = O - U (L148)
          const float P = __fmaf_rn(L.x, E, -NU[x]);                         // preliminary (L178)
          const float mxf = add_f32_f16(mx_h, 0.0f), mnf = add_f32_f16(mn_h, 0.0f);
          const float t = fminf(fmaxf(P, mnf), mxf);                         // Fig. 8 branch target
          F8[x] = __fmaf_rn(L.y, __fsub_rn(P, t), t);                        // osc max / osc min / P
        }
        // clamp [0,255] + RNE (R14) or truncation (the R14 alternative), packed 4 per word
        const uint32_t o0 = trunc ? pack4_rzi_u8(F8[0], F8[1], F8[2], F8[3]) : pack4_rni_u8(F8[0], F8[1], F8[2], F8[3]);
        const uint32_t o1 = trunc ? pack4_rzi_u8(F8[4], F8[5], F8[6], F8[7]) : pack4_rni_u8(F8[4], F8[5], F8[6], F8[7]);
        uint8_t *orow = out + (size_t)r * W;
        if (c0 < W) *reinterpret_cast<uint32_t *>(orow + c0) = o0;
        if (c0 + 4 < W) *reinterpret_cast<uint32_t *>(orow + c0 + 4) = o1;
      }
      ra = rb;
      rb = rc;
    }
    prev = cur;
    cur = next;
  }
}

}  // namespace

static void geometry(int W, int H, int &tiles_x, int &tiles_y, int &ctas) {
  tiles_x = (W + kWarpCols - 1) / kWarpCols;
  tiles_y = (H + kTileRows - 1) / kTileRows;
  ctas = (tiles_x * tiles_y + kWarps - 1) / kWarps;
}

cudaError_t launch_edge_sum(const uint8_t *imgs, int n, int W, int H, const Params &p,
                            unsigned long long *sums, unsigned int *counters, float2 *luts,
                            double *means, cudaStream_t stream) {
  int tx, ty, ctas;
  geometry(W, H, tx, ty, ctas);
  edge_sum_kernel<<<dim3(ctas, n), kThreads, 0, stream>>>(imgs, W, H, tx, ty, p, sums, counters, luts, means);
  return cudaGetLastError();
}

cudaError_t launch_sharpen(const uint8_t *imgs, int n, int W, int H, const float2 *luts, uint8_t *outs, int flags,
                           cudaStream_t stream) {
  int tx, ty, ctas;
  geometry(W, H, tx, ty, ctas);
  sharpen_kernel<<<dim3(ctas, n), kThreads, 0, stream>>>(imgs, W, H, tx, ty, luts, outs, flags);
  return cudaGetLastError();
}

// Forces the (lazy) module load of this file's kernels; see kernels.h.
cudaError_t preload_two_pass() {
  cudaFuncAttributes a;
  cudaError_t e;
  if ((e = cudaFuncGetAttributes(&a, edge_sum_kernel)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, sharpen_kernel)) != cudaSuccess) return e;
  return cudaSuccess;
}

}  // namespace sharp
