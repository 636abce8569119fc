// TMA-staged persistent sm_100a kernels (the main path; needs W % 16 == 0
// and a 16-byte aligned frame base -- the TMA tensor-map rules).
//
// Work unit ("task"): a CTA tile of 4 warp tiles side by side, each warp tile
// 240 output columns x 32 output rows of one frame.  Each warp's tile plus
// halo (256 columns: 8 left, 8 right; 4 rows above/below for pass 2, 1 for
// pass 1) is fetched by one cp.async.bulk.tensor (TMA) 3-D box load into
// shared memory; out-of-image pixels are zero-filled by the TMA unit, so
// there are no bounds checks in the pixel loops.  CTAs are persistent over
// a contiguous range of tasks and double-buffer: task i+1's boxes (and its
// frame's lookup table, pass 2) are in flight while task i is computed.
//
// Interior code handles every pixel with the body formulas; the image
// border is handled by
//   * rows 0, 1, H-2, H-1: a warp-uniform branch (upscale border lines of
//     L140, Sobel frame L160, overshoot frame L208);
//   * columns 0, 1, W-2, W-1: a specialised border pass of the warps whose
//     tile touches them, recomputing those pixels with the scalar rules
//     (sec. V-E "border optimization", on the GPU at every size).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <algorithm>
#include <stdint.h>

#include "device_common.cuh"
#include "kernels.h"

namespace sharp {
namespace {
using namespace dev;

constexpr int kTW = 240;            // output columns per warp tile (30 lanes x 8 px)
constexpr int kTH = 32;             // output rows per warp tile
constexpr int kWarpsT = 4;          // warps (warp tiles) per CTA tile
constexpr int kCtaCols = kTW * kWarpsT;
constexpr int kThreadsT = 32 * kWarpsT;
// The TMA box's innermost start coordinate must be 16-byte aligned, and a
// box dimension is at most 256 elements, so the frames are viewed as 4-D
// [n][H][W/16][16] and a warp tile's box is {16, 17 chunks, rows, 1}: 272
// columns starting at C0w-16 (16-aligned), i.e. an smem row pitch of 272.
constexpr int kChunks = 17;
constexpr int kPitch = 16 * kChunks;  // 272: smem columns C0w-16 .. C0w+255
constexpr int kCol0 = 16;             // smem column of C0w
constexpr int kRows2 = kTH + 8;       // pass 2 box rows (R0-4 .. R0+35)
constexpr int kRows1 = kTH + 2;       // pass 1 box rows (R0-1 .. R0+32)
constexpr int kBox2 = kPitch * kRows2;                  // 10880 = 85 * 128
constexpr int kBox1 = (kPitch * kRows1 + 127) / 128 * 128;  // 9344 (smem destinations 128-B aligned)
static_assert(kBox2 % 128 == 0, "TMA smem destination alignment");
constexpr int kLutBytes = kLutSize * 8;
constexpr int kSmem2 = 2 * (kWarpsT * kBox2 + kLutBytes) + 64;
constexpr int kSmem1 = 2 * kWarpsT * kBox1 + 64;

// ------------------------------------------------------------ TMA / mbarrier
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
// Box of the warp tile whose first output column is C0w (multiple of 16):
// columns C0w-16 .. C0w+255, rows r .. r+box_rows-1 of frame f.
__device__ __forceinline__ void tma_box(uint32_t dst, const CUtensorMap *map, int C0w, int r, int f, uint32_t bar) {
  const int chunk = (C0w - kCol0) / 16;
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], "
      "[%6];" ::"r"(dst),
      "l"(map), "r"(0), "r"(chunk), "r"(r), "r"(f), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void bulk_copy(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_barrier_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void prefetch_map(const CUtensorMap *m) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(m) : "memory");
}

struct TaskGeom {
  int W, H;
  int tiles_x;    // CTA tiles per row band (ceil(W / 960))
  int tiles_y;    // row bands (ceil(H / 32))
  int per_frame;  // tiles_x * tiles_y
  int ntasks;     // per_frame * n
};

__device__ __forceinline__ void task_coords(const TaskGeom &g, int t, int &f, int &C0, int &R0) {
  f = t / g.per_frame;
  const int rem = t - f * g.per_frame;
  const int ty = rem / g.tiles_x;
  C0 = (rem - ty * g.tiles_x) * kCtaCols;
  R0 = ty * kTH;
}

// Words of smem row `s` for this lane (addresses precomputed per lane).
struct LaneAddr {
  uint32_t w, p, n;  // w0w1 (8 B), pw, nw
};
__device__ __forceinline__ Words lds_words(const LaneAddr &a, int s) {
  const uint32_t off = (uint32_t)s * kPitch;
  const uint2 w = lds_u64(a.w + off);
  return Words{lds_u32(a.p + off), w.x, w.y, lds_u32(a.n + off)};
}

// D sums (16*D) of the 4-row block starting at smem row s for D columns
// j0-1, j0, j0+1, j0+2 of this lane.  Own columns from the lane's words;
// the neighbours by shuffle (lane 31 supplies the left halo column of the
// warp tile, lane 30 the right one).
__device__ __forceinline__ float4 dblock(uint32_t ad0, uint32_t ad1, int s, int lane) {
  const uint32_t off = (uint32_t)s * kPitch;
  const uint32_t s0 = blk4(lds_u32(ad0 + off), lds_u32(ad0 + off + kPitch), lds_u32(ad0 + off + 2 * kPitch),
                           lds_u32(ad0 + off + 3 * kPitch));
  const uint32_t s1 = blk4(lds_u32(ad1 + off), lds_u32(ad1 + off + kPitch), lds_u32(ad1 + off + 2 * kPitch),
                           lds_u32(ad1 + off + 3 * kPitch));
  const float d0 = (float)s0, d1 = (float)s1;
  const float dm1 = __shfl_sync(0xffffffffu, d1, (lane + 31) & 31);
  const float d2 = __shfl_sync(0xffffffffu, d0, (lane + 1) & 31);
  return make_float4(dm1, d0, d1, d2);
}

// ------------------------------------------------------- scalar border pixel
// 16*D of block (i, j) read from the warp's smem tile (rows R0-4.., cols C0w-8..).
__device__ __forceinline__ float dsum_at(uint32_t tile, int i, int j, int R0, int C0w) {
  const uint32_t a = tile + (uint32_t)(4 * i - R0 + 4) * kPitch + (uint32_t)(4 * j - C0w + kCol0);
  return (float)blk4(lds_u32(a), lds_u32(a + kPitch), lds_u32(a + 2 * kPitch), lds_u32(a + 3 * kPitch));
}

// U at (r, c), any pixel (body formula of L146 or the border rules of
// L140-L142, last writer of steps i..vii), from the smem tile.
__device__ float u_any(uint32_t tile, int r, int c, int W, int H, int R0, int C0w) {
  const int w = W >> 2, h = H >> 2;
  const bool ring = r < 2 || r >= H - 2 || c < 2 || c >= W - 2;
  if (!ring) {
    const int i = (r - 2) >> 2, a = (r - 2) & 3, j = (c - 2) >> 2, b = (c - 2) & 3;
    const float wt = (float)wt_of((a + 2) & 3), wl = (float)wl_of((b + 2) & 3);
    // rows: a = 0..3 -> weights (7,1),(5,3),(3,5),(1,7) == wt_of(a+2)
    const float v0 = __fmaf_rn(8.0f - wt, dsum_at(tile, i + 1, j, R0, C0w), __fmul_rn(wt, dsum_at(tile, i, j, R0, C0w)));
    const float v1 =
        __fmaf_rn(8.0f - wt, dsum_at(tile, i + 1, j + 1, R0, C0w), __fmul_rn(wt, dsum_at(tile, i, j + 1, R0, C0w)));
    return __fmaf_rn((8.0f - wl) * (1.0f / 1024.0f), v1, __fmul_rn(wl * (1.0f / 1024.0f), v0));
  }
  if (r >= H - 2 && c >= W - 2) return __fmul_rn(dsum_at(tile, h - 1, w - 1, R0, C0w), 1.0f / 16.0f);  // (vii)
  if ((c <= 1 || c >= W - 2) && r <= H - 3) {                                                             // columns
    const int j = (c <= 1) ? 0 : w - 1;
    if (c <= 1 && r <= 1) return __fmul_rn(dsum_at(tile, 0, 0, R0, C0w), 1.0f / 16.0f);  // (v) then (vi)
    const int rr = (r == H - 3) ? H - 4 : r;  // third last <- fourth last
    const int i = rr >> 2, k = rr & 3;
    const float x = dsum_at(tile, i, j, R0, C0w);
    return k == 0 ? __fmul_rn(x, 1.0f / 16.0f) : line_val(x, dsum_at(tile, i + 1, j, R0, C0w), k);
  }
  // rows 0/1 (line of D row 0) or H-2/H-1 (line of D row h-1)
  const int i = (r <= 1) ? 0 : h - 1;
  const int cc = (c == W - 3) ? W - 4 : c;
  const int j = cc >> 2, k = cc & 3;
  const float x = dsum_at(tile, i, j, R0, C0w);
  return k == 0 ? __fmul_rn(x, 1.0f / 16.0f) : line_val(x, dsum_at(tile, i, j + 1, R0, C0w), k);
}

// The whole pipeline for one pixel with scalar code (specialised border pass).
__device__ uint32_t pixel_generic(uint32_t tile, uint32_t lut, int r, int c, int W, int H, int R0, int C0w) {
  const uint32_t base = tile + (uint32_t)(r - R0 + 4) * kPitch + (uint32_t)(c - C0w + kCol0);
  const int o = (int)lds_u8(base);
  int pe = 0, mx = 255, mn = 0;
  if (!(r == 0 || r == H - 1 || c == 0 || c == W - 1)) {  // Sobel frame (L160) / overshoot frame (L208)
    int v[3][3];
#pragma unroll
    for (int u = 0; u < 3; ++u)
#pragma unroll
      for (int q = 0; q < 3; ++q) v[u][q] = (int)lds_u8(base + (uint32_t)((u - 1) * kPitch + (q - 1)));
    const int gx = (v[0][2] + 2 * v[1][2] + v[2][2]) - (v[0][0] + 2 * v[1][0] + v[2][0]);
    const int gy = (v[2][0] + 2 * v[2][1] + v[2][2]) - (v[0][0] + 2 * v[0][1] + v[0][2]);
    pe = abs(gx) + abs(gy);
    mx = 0;
    mn = 255;
#pragma unroll
    for (int u = 0; u < 3; ++u)
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        mx = max(mx, v[u][q]);
        mn = min(mn, v[u][q]);
      }
  }
  const float U = u_any(tile, r, c, W, H, R0, C0w);
  const float2 L = lds_f2(lut + 8u * (uint32_t)pe);
  const float E = __fsub_rn((float)o, U);
  return sharpen_px(L.x, L.y, E, U, (float)mx, (float)mn);
}

// ======================================================== pass 2 (per warp)
__device__ __forceinline__ void p2_warp(uint32_t tile, uint32_t lut, uint8_t *__restrict__ out, int W, int H, int C0w,
                                        int R0, int lane) {
  const int c0 = C0w + 8 * lane;
  const bool active = lane < 30 && c0 < W;
  const int ll = lane < 30 ? lane : 0;  // idle lanes read lane 0's words (results unused)
  const LaneAddr A{tile + kCol0 + 8u * ll, tile + kCol0 - 4u + 8u * ll, tile + kCol0 + 8u + 8u * ll};
  const uint32_t ad0 = tile + (lane == 30 ? kCol0 + 240u : kCol0 + 8u * ll);     // lane 30: right halo D column
  const uint32_t ad1 = tile + (lane == 31 ? kCol0 - 4u : kCol0 + 4u + 8u * ll);  // lane 31: left halo D column
  // LDS address of {adj, osc}[p] from the bits of (2^23 + p) as f32: q*8 + base'.
  const uint32_t lut_q = lut - (0x4B000000u << 3);
  const int rend = min(R0 + kTH, H);

  float4 Dp = dblock(ad0, ad1, 0, lane);  // D row k0-1 (smem rows 0..3)
  float4 Dc = dblock(ad0, ad1, 4, lane);  // D row k0
  RowD ra = derive<true>(lds_words(A, 3));
  RowD rb = derive<true>(lds_words(A, 4));
  uint8_t *orow = out + (size_t)R0 * W + c0;

#pragma unroll 1
  for (int j = 0; j < kTH / 4; ++j) {
    if (R0 + 4 * j >= rend) break;
    const float4 Dn = dblock(ad0, ad1, 8 + 4 * j, lane);  // D row k+1
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      const int r = R0 + 4 * j + a;
      if (r >= rend) break;
      const RowD rc = derive<true>(lds_words(A, 4 * j + a + 5));
      uint32_t pe[4], MX[4], MN[4];
      sobel(ra, rb, rc, pe);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        MX[i] = __vimax3_u16x2(ra.mx[i], rb.mx[i], rc.mx[i]);
        MN[i] = __vimin3_u16x2(ra.mn[i], rb.mn[i], rc.mn[i]);
      }
      // Upscale body (L146): vertical interpolation of the four D columns,
      // then horizontal, as -U (exact).  a' = 0,1 -> D rows (k-1, k),
      // a' = 2,3 -> (k, k+1).
      const float wt = (float)wt_of(a), wb = 8.0f - wt;
      const float4 T = a < 2 ? Dp : Dc, B = a < 2 ? Dc : Dn;
      const float V[4] = {__fmaf_rn(wb, B.x, __fmul_rn(wt, T.x)), __fmaf_rn(wb, B.y, __fmul_rn(wt, T.y)),
                          __fmaf_rn(wb, B.z, __fmul_rn(wt, T.z)), __fmaf_rn(wb, B.w, __fmul_rn(wt, T.w))};
      float NU[8];
#pragma unroll
      for (int x = 0; x < 8; ++x) {
        const float wl = (float)wl_of(x);
        NU[x] = __fmaf_rn(-(8.0f - wl) * (1.0f / 1024.0f), V[jl_of(x) + 1], __fmul_rn(-wl * (1.0f / 1024.0f), V[jl_of(x)]));
      }
      if (r < 2 || r >= H - 2) {  // border rows (warp-uniform)
        // Upscale border lines (L140): rows 0,1 from D row 0, rows H-2,H-1
        // from D row h-1 (== Dc here); columns 0,1,W-2,W-1 are redone by the
        // border pass below.
        const float q[4] = {Dc.y, Dc.z, Dc.w, Dc.w};
#pragma unroll
        for (int x = 0; x < 8; ++x) {
          const int c = c0 + x;
          const int cc = (c == W - 3) ? c - 1 : c;
          const int jx = (cc - c0) >> 2, k = cc & 3;
          NU[x] = -(k == 0 ? __fmul_rn(q[jx], 1.0f / 16.0f) : line_val(q[jx], q[jx + 1], k));
        }
        if (r == 0 || r == H - 1) {  // frame: Sobel 0, no overshoot window
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            pe[i] = 0u;
            MX[i] = kF16_255 | (kF16_255 << 16);
            MN[i] = 0u;
          }
        }
      }
      uint32_t o[8];
#pragma unroll
      for (int x = 0; x < 8; ++x) {
        const int p = pair_of(x);
        const bool hi = half_of(x);
        const uint16_t pe_h = hi ? hi16(pe[p]) : lo16(pe[p]);
        const uint32_t qb = __float_as_uint(add_f32_f16(pe_h, 8388608.0f));  // 2^23 + pEdge
        const float2 L = lds_f2(qb * 8u + lut_q);                           // {adj, osc}
        const float E = add_f32_f16(hi ? hi16(rb.c[p]) : lo16(rb.c[p]), NU[x]);  // pError = O - U (L148)
        const float mxf = add_f32_f16(hi ? hi16(MX[p]) : lo16(MX[p]), 0.0f);
        const float mnf = add_f32_f16(hi ? hi16(MN[p]) : lo16(MN[p]), 0.0f);
        o[x] = sharpen_px(L.x, L.y, E, -NU[x], mxf, mnf);
      }
      if (active) *reinterpret_cast<uint2 *>(orow) = pack8(o);
      orow += W;
      ra = rb;
      rb = rc;
    }
    Dp = Dc;
    Dc = Dn;
  }

  // Specialised border pass: columns 0,1 and W-2,W-1 of this tile.
  const bool left = (C0w == 0), right = (C0w <= W - 2 && W - 2 < C0w + kTW);
  if (left || right) {
    __syncwarp();
    const int nr = rend - R0;
    const int ncol = (left ? 2 : 0) + (right ? 2 : 0);
    for (int idx = lane; idx < nr * ncol; idx += 32) {
      const int r = R0 + idx / ncol;
      const int k = idx % ncol;  // left: 0,1 -> columns 0,1; then W-2, W-1
      const int c = left ? (k < 2 ? k : W - 4 + k) : W - 2 + k;
      out[(size_t)r * W + c] = (uint8_t)pixel_generic(tile, lut, r, c, W, H, R0, C0w);
    }
  }
}

__global__ void __launch_bounds__(kThreadsT) sharpen_tma_kernel(const __grid_constant__ CUtensorMap tmap,
                                                                 const float2 *__restrict__ luts,
                                                                 uint8_t *__restrict__ outs, TaskGeom g) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar0 = sbase + 2 * (kWarpsT * kBox2 + kLutBytes);
  auto buf_tile = [&](int b, int w) { return sbase + (uint32_t)(b * (kWarpsT * kBox2 + kLutBytes) + w * kBox2); };
  auto buf_lut = [&](int b) { return sbase + (uint32_t)(b * (kWarpsT * kBox2 + kLutBytes) + kWarpsT * kBox2); };

  const int t0 = (int)(((long long)blockIdx.x * g.ntasks) / gridDim.x);
  const int t1 = (int)(((long long)(blockIdx.x + 1) * g.ntasks) / gridDim.x);
  if (threadIdx.x == 0) {
    prefetch_map(&tmap);
    mbar_init(bar0, 1);
    mbar_init(bar0 + 8, 1);
    fence_barrier_init();
  }
  __syncthreads();

  auto issue = [&](int t, int b) {
    int f, C0, R0;
    task_coords(g, t, f, C0, R0);
    int nw = 0;
    for (int w = 0; w < kWarpsT; ++w) nw += (C0 + w * kTW < g.W);
    const uint32_t bar = bar0 + 8u * b;
    fence_proxy_async();
    mbar_expect_tx(bar, (uint32_t)(nw * kBox2 + kLutBytes));
    for (int w = 0; w < nw; ++w) tma_box(buf_tile(b, w), &tmap, C0 + w * kTW, R0 - 4, f, bar);
    bulk_copy(buf_lut(b), luts + (size_t)f * kLutSize, kLutBytes, bar);
  };

  if (threadIdx.x == 0 && t0 < t1) issue(t0, 0);
  for (int t = t0, i = 0; t < t1; ++t, ++i) {
    const int b = i & 1;
    __syncthreads();  // everyone is done with buffer b^1 (task t-1)
    if (threadIdx.x == 0 && t + 1 < t1) issue(t + 1, b ^ 1);
    mbar_wait(bar0 + 8u * b, (uint32_t)((i >> 1) & 1));
    int f, C0, R0;
    task_coords(g, t, f, C0, R0);
    const int C0w = C0 + warp * kTW;
    if (C0w < g.W)
      p2_warp(buf_tile(b, warp), buf_lut(b), outs + (size_t)f * g.W * g.H, g.W, g.H, C0w, R0, lane);
  }
}

// ======================================================== pass 1 (per warp)
__device__ __forceinline__ float p1_warp(uint32_t tile, int W, int H, int C0w, int R0, int lane) {
  const int c0 = C0w + 8 * lane;
  const int ll = lane < 30 ? lane : 0;
  const LaneAddr A{tile + kCol0 + 8u * ll, tile + kCol0 - 4u + 8u * ll, tile + kCol0 + 8u + 8u * ll};
  const int rend = min(R0 + kTH, H);
  // Pixels of this lane that belong to the Sobel body (not the frame columns,
  // not beyond the image): lanes at the image's left/right edge only.
  uint32_t vmask = 0;
#pragma unroll
  for (int x = 0; x < 8; ++x) vmask |= (uint32_t)(c0 + x >= 1 && c0 + x <= W - 2) << x;
  const bool edge = vmask != 0xffu;
  RowD ra = derive<false>(lds_words(A, 0));
  RowD rb = derive<false>(lds_words(A, 1));
  float acc = 0.0f;  // exact: < 8 px * 32 rows * 1530 < 2^24
#pragma unroll 4
  for (int r = R0; r < rend; ++r) {
    const RowD rc = derive<false>(lds_words(A, r - R0 + 2));
    uint32_t pe[4];
    sobel(ra, rb, rc, pe);
    if (r != 0 && r != H - 1) {  // Sobel border rows are 0 (L160)
      if (!edge) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          acc = add_f32_f16(lo16(pe[i]), acc);
          acc = add_f32_f16(hi16(pe[i]), acc);
        }
      } else {
#pragma unroll
        for (int x = 0; x < 8; ++x)
          if (vmask >> x & 1) acc = add_f32_f16(half_of(x) ? hi16(pe[pair_of(x)]) : lo16(pe[pair_of(x)]), acc);
      }
    }
    ra = rb;
    rb = rc;
  }
  return (lane < 30) ? acc : 0.0f;
}

__global__ void __launch_bounds__(kThreadsT) edge_sum_tma_kernel(const __grid_constant__ CUtensorMap tmap, TaskGeom g,
                                                                  Params prm, unsigned long long *__restrict__ sums,
                                                                  unsigned int *__restrict__ counters,
                                                                  float2 *__restrict__ luts, double *__restrict__ means) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint32_t warp_sum[kWarpsT];
  __shared__ int last_frame;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar0 = sbase + 2 * kWarpsT * kBox1;
  auto buf_tile = [&](int b, int w) { return sbase + (uint32_t)((b * kWarpsT + w) * kBox1); };

  const int t0 = (int)(((long long)blockIdx.x * g.ntasks) / gridDim.x);
  const int t1 = (int)(((long long)(blockIdx.x + 1) * g.ntasks) / gridDim.x);
  if (threadIdx.x == 0) {
    prefetch_map(&tmap);
    mbar_init(bar0, 1);
    mbar_init(bar0 + 8, 1);
    fence_barrier_init();
  }
  __syncthreads();
  auto issue = [&](int t, int b) {
    int f, C0, R0;
    task_coords(g, t, f, C0, R0);
    int nw = 0;
    for (int w = 0; w < kWarpsT; ++w) nw += (C0 + w * kTW < g.W);
    const uint32_t bar = bar0 + 8u * b;
    fence_proxy_async();
    mbar_expect_tx(bar, (uint32_t)(nw * kPitch * kRows1));
    for (int w = 0; w < nw; ++w) tma_box(buf_tile(b, w), &tmap, C0 + w * kTW, R0 - 1, f, bar);
  };
  if (threadIdx.x == 0 && t0 < t1) issue(t0, 0);
  for (int t = t0, i = 0; t < t1; ++t, ++i) {
    const int b = i & 1;
    __syncthreads();
    if (threadIdx.x == 0 && t + 1 < t1) issue(t + 1, b ^ 1);
    mbar_wait(bar0 + 8u * b, (uint32_t)((i >> 1) & 1));
    int f, C0, R0;
    task_coords(g, t, f, C0, R0);
    const int C0w = C0 + warp * kTW;
    float acc = 0.0f;
    if (C0w < g.W) acc = p1_warp(buf_tile(b, warp), g.W, g.H, C0w, R0, lane);
    // Reduction stage 1 (sec. V-C): warp reduction, CTA partial, u64 atomic.
    const uint32_t ws = __reduce_add_sync(0xffffffffu, (uint32_t)acc);
    if (lane == 0) warp_sum[warp] = ws;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long part = 0;
#pragma unroll
      for (int w = 0; w < kWarpsT; ++w) part += warp_sum[w];
      atomicAdd(&sums[f], part);
      __threadfence();
      const unsigned int ticket = atomicAdd(&counters[f], 1u);
      last_frame = (ticket == (unsigned)g.per_frame - 1) ? f : -1;
    }
    __syncthreads();
    const int lf = last_frame;
    if (lf >= 0) {
      // Stage 2, last-block-done: mean and the frame's lookup tables.
      __threadfence();
      const unsigned long long S = atomicAdd(&sums[lf], 0ull);
      const double mean = (double)S / ((double)g.W * (double)g.H);
      const double m = mean > 1.0 ? mean : 1.0;
      for (int p = threadIdx.x; p < kLutSize; p += kThreadsT) {
        float adj = 0.0f, osc = 0.0f;
        if (p <= 1530) {
          adj = (float)((double)prm.amount * pow((double)p / m, (double)prm.gamma));
          osc = (float)fmin(fmax((double)prm.osc_gain * exp(-(double)p / ((double)prm.osc_scale * m)), 0.0), 1.0);
        }
        luts[(size_t)lf * kLutSize + p] = make_float2(adj, osc);
      }
      if (threadIdx.x == 0) {
        means[lf] = mean;
        counters[lf] = 0u;  // re-arm for the next launch
      }
    }
  }
}

// ----------------------------------------------------------------- host side
PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void *p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
  }
  return fn;
}

bool make_map(CUtensorMap *m, const uint8_t *imgs, int n, int W, int H, int box_rows) {
  auto fn = encode_fn();
  if (!fn) return false;
  // [n][H][W/16][16] view (see kChunks).
  const cuuint64_t dims[4] = {16, (cuuint64_t)W / 16, (cuuint64_t)H, (cuuint64_t)n};
  const cuuint64_t strides[3] = {16, (cuuint64_t)W, (cuuint64_t)W * H};
  const cuuint32_t box[4] = {16, (cuuint32_t)kChunks, (cuuint32_t)box_rows, 1};
  const cuuint32_t estr[4] = {1, 1, 1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, (void *)imgs, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

TaskGeom geom(int n, int W, int H) {
  TaskGeom g;
  g.W = W;
  g.H = H;
  g.tiles_x = (W + kCtaCols - 1) / kCtaCols;
  g.tiles_y = (H + kTH - 1) / kTH;
  g.per_frame = g.tiles_x * g.tiles_y;
  g.ntasks = g.per_frame * n;
  return g;
}

int num_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

}  // namespace

bool tma_supported(const uint8_t *imgs, const uint8_t *outs, int W, int H) {
  return (W % 16) == 0 && (((uintptr_t)imgs) & 15) == 0 && (((uintptr_t)outs) & 7) == 0 && H >= 8 &&
         encode_fn() != nullptr;
}

cudaError_t launch_edge_sum_tma(const uint8_t *imgs, int n, int W, int H, const Params &p, unsigned long long *sums,
                                unsigned int *counters, float2 *luts, double *means, cudaStream_t stream) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(edge_sum_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem1);
    attr = true;
  }
  CUtensorMap m;
  if (!make_map(&m, imgs, n, W, H, kRows1)) return cudaErrorInvalidValue;
  const TaskGeom g = geom(n, W, H);
  const int grid = std::min(g.ntasks, 3 * num_sms());
  edge_sum_tma_kernel<<<grid, kThreadsT, kSmem1, stream>>>(m, g, p, sums, counters, luts, means);
  return cudaGetLastError();
}

cudaError_t launch_sharpen_tma(const uint8_t *imgs, int n, int W, int H, const float2 *luts, uint8_t *outs,
                               cudaStream_t stream) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(sharpen_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem2);
    attr = true;
  }
  CUtensorMap m;
  if (!make_map(&m, imgs, n, W, H, kRows2)) return cudaErrorInvalidValue;
  const TaskGeom g = geom(n, W, H);
  const int grid = std::min(g.ntasks, 2 * num_sms());
  sharpen_tma_kernel<<<grid, kThreadsT, kSmem2, stream>>>(m, luts, outs, g);
  return cudaGetLastError();
}

}  // namespace sharp
