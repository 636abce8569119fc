// TMA-staged, dynamically scheduled sm_100a "step" kernel (the main path;
// needs W % 16 == 0 and 16-byte aligned frames -- the TMA tensor-map rules).
//
// One launch runs two kinds of tasks, grabbed in order from a global counter
// by persistent CTAs (2 per SM):
//   * pass-1 tasks of chunk c+1: Sobel (L158-L172) + reduction (L174, sec.
//     V-C); the CTA finishing a frame's last pass-1 task computes the frame's
//     mean and lookup tables (last-block-done);
//   * pass-2 tasks of chunk c: the fused per-pixel pipeline (downscale L130,
//     upscale L140-L146, pError L148, Sobel, 3x3 max/min L182, strength L178,
//     preliminary L178, overshoot L180-L212) -> u8.
// Pass-1 tasks come first, so the frames' table builds overlap the pass-2
// tasks of other CTAs, and the chunk's input is re-read from L2 by pass 2 in
// the next launch.
//
// A task is a CTA tile of 4 warp tiles side by side; a warp tile is 240
// output columns x 24 rows of one frame.  Its pixels plus halo are fetched by
// one cp.async.bulk.tensor (TMA) box into shared memory (out-of-image pixels
// are zero-filled by the TMA unit: no bounds checks in the pixel loops), and
// the next task's boxes are in flight while the current one is computed.
// Each lane owns 8 adjacent columns and walks down the rows with a 3-row
// window; the row loop is unrolled 12 rows (lcm of the 3-row window and the
// 4-row downscale block) so the window never needs register moves.  Lanes 30
// and 31 fetch the right/left halo columns and hand them out by shuffle.
//
// Image border: rows 0,1,H-2,H-1 by a warp-uniform branch; columns 0,1,W-2,
// W-1 by a specialised scalar pass of the warps whose tile touches them.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>

#include "device_common.cuh"
#include "kernels.h"

namespace sharp {
namespace {
using namespace dev;

constexpr int kTW = 240;     // output columns per warp tile (lanes 0..29 x 8 px)
constexpr int kTH = 24;      // output rows per warp tile (two 12-row bodies)
constexpr int kWarpsT = 4;   // warp tiles per CTA tile
constexpr int kCtaCols = kTW * kWarpsT;
constexpr int kThreadsT = 32 * kWarpsT;
// The TMA box's innermost start coordinate must be 16-byte aligned and a box
// dimension is at most 256, so frames are viewed as 4-D [n][H][W/16][16] and
// a warp tile's box is {16, 17 chunks, rows, 1}: 272 columns from C0w-16.
constexpr int kChunks = 17;
constexpr int kPitch = 16 * kChunks;  // smem row pitch: columns C0w-16 .. C0w+255
constexpr int kCol0 = 16;             // smem column of C0w
constexpr int kRows2 = kTH + 8;       // pass-2 box rows: R0-4 .. R0+27
constexpr int kRows1 = kTH + 2;       // pass-1 box rows: R0-1 .. R0+24
constexpr int kBox2 = kPitch * kRows2;  // 8704 = 68 * 128
constexpr int kBox1 = kPitch * kRows1;  // 7072
constexpr int kSlot = kBox2;            // per-warp smem slot (128-B aligned)
constexpr int kLutBytes = kLutSize * 8;
constexpr int kStage = kWarpsT * kSlot + kLutBytes;
constexpr int kSmem = 2 * kStage + 64;
static_assert(kSlot % 128 == 0 && kStage % 128 == 0, "TMA smem destinations must be 128-B aligned");
static_assert(kTH % 12 == 0, "row loop is unrolled by 12");

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
// Box of the warp tile whose first output column is C0w (a multiple of 16):
// columns C0w-16 .. C0w+255, rows r .. r+rows-1 of frame f.
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

// ----------------------------------------------------------- packed f32x2
__device__ __forceinline__ unsigned long long f2pack(float a, float b) {
  unsigned long long r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ float2 f2unpack(unsigned long long r) {
  float2 v;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(v.x), "=f"(v.y) : "l"(r));
  return v;
}
// (a*x + b*y) for a lane pair with the same (x, y): two single-rounding ops
// (FMUL2 then FFMA2), bit-identical to the scalar fmul/fma pair.
__device__ __forceinline__ float2 lin2(float x, float y, float a0, float a1, float b0, float b1) {
  unsigned long long t, r;
  const unsigned long long xx = f2pack(x, x), yy = f2pack(y, y);
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(t) : "l"(xx), "l"(f2pack(a0, a1)));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(yy), "l"(f2pack(b0, b1)), "l"(t));
  return f2unpack(r);
}
__device__ __forceinline__ float2 sub2(float2 a, float2 b) {
  unsigned long long r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(f2pack(a.x, a.y)), "l"(f2pack(b.x, b.y)));
  return f2unpack(r);
}

// ------------------------------------------------------------------ tasks
struct Geo {
  int W, H;
  int tiles_x;    // CTA tiles per row band (ceil(W / 960))
  int per_frame;  // CTA tiles per frame
};
__device__ __forceinline__ void tile_of(const Geo &g, int t, int &f, int &C0, int &R0) {
  f = t / g.per_frame;
  const int rem = t - f * g.per_frame;
  const int ty = rem / g.tiles_x;
  C0 = (rem - ty * g.tiles_x) * kCtaCols;
  R0 = ty * kTH;
}

struct StepParams {
  Geo g;
  int n1, n2;  // pass-1 / pass-2 task counts
  Params prm;
  unsigned long long *sums1;
  double *means1;
  unsigned int *counters1;
  float2 *luts1;
  const float2 *luts2;
  uint8_t *out2;
  unsigned int *task_counter;
};

// ------------------------------------------------------------- row window
// Lane words of smem row s: lanes 0..29 own columns C0w+8l..+7; lane 30 the
// right halo C0w+240..247, lane 31 the left halo C0w-8..C0w-1.
__device__ __forceinline__ uint2 row_words(uint32_t a, int s) { return lds_u64(a + (uint32_t)s * kPitch); }

// Converts a row of words into the window data.  Neighbour pairs come from
// the adjacent lanes (shuffle), so each lane loads only its own 8 bytes.
template <bool kMinMax>
__device__ __forceinline__ RowD derive_w(uint2 w, int lane) {
  const uint32_t E0 = hadd(prmt(w.x, kF16Bias, 0x4240), kMinus1024);  // (c0, c0+2)
  const uint32_t O0 = hadd(prmt(w.x, kF16Bias, 0x4341), kMinus1024);  // (c0+1, c0+3)
  const uint32_t E1 = hadd(prmt(w.y, kF16Bias, 0x4240), kMinus1024);  // (c0+4, c0+6)
  const uint32_t O1 = hadd(prmt(w.y, kF16Bias, 0x4341), kMinus1024);  // (c0+5, c0+7)
  const uint32_t PO = __shfl_sync(0xffffffffu, O1, (lane + 31) & 31);  // (c0-3, c0-1)
  const uint32_t NE = __shfl_sync(0xffffffffu, E0, (lane + 1) & 31);   // (c0+8, c0+10)
  const uint32_t p[4] = {E0, O0, E1, O1};
  const uint32_t l[4] = {prmt(PO, O0, 0x5432), E0, prmt(O0, O1, 0x5432), E1};
  const uint32_t r[4] = {O0, prmt(E0, E1, 0x5432), O1, prmt(E1, NE, 0x5432)};
  RowD d;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    d.c[i] = p[i];
    d.h[i] = hsub(r[i], l[i]);
    d.s[i] = hadd(hfma(kTwo, p[i], l[i]), r[i]);
    if (kMinMax) {
      d.mx[i] = __vimax3_u16x2(l[i], p[i], r[i]);
      d.mn[i] = __vimin3_u16x2(l[i], p[i], r[i]);
    }
  }
  return d;
}

// D sums (16*D) of the block at smem rows s..s+3 for D columns j0-1..j0+2.
__device__ __forceinline__ float4 dblock(uint32_t a, int s, int lane) {
  const uint32_t o = a + (uint32_t)s * kPitch;
  const uint2 r0 = lds_u64(o), r1 = lds_u64(o + kPitch), r2 = lds_u64(o + 2 * kPitch), r3 = lds_u64(o + 3 * kPitch);
  const float d0 = (float)blk4(r0.x, r1.x, r2.x, r3.x);
  const float d1 = (float)blk4(r0.y, r1.y, r2.y, r3.y);
  const float dm1 = __shfl_sync(0xffffffffu, d1, (lane + 31) & 31);
  const float d2 = __shfl_sync(0xffffffffu, d0, (lane + 1) & 31);
  return make_float4(dm1, d0, d1, d2);
}

// ------------------------------------------------------- scalar border pixel
__device__ __forceinline__ float dsum_at(uint32_t tile, int i, int j, int R0, int C0w) {
  const uint32_t a = tile + (uint32_t)(4 * i - R0 + 4) * kPitch + (uint32_t)(4 * j - C0w + kCol0);
  return (float)blk4(lds_u32(a), lds_u32(a + kPitch), lds_u32(a + 2 * kPitch), lds_u32(a + 3 * kPitch));
}

// U at (r, c), any pixel: body formula of L146 or the border rules of
// L140-L142 (the last writer of steps i..vii), from the smem tile.
__device__ float u_any(uint32_t tile, int r, int c, int W, int H, int R0, int C0w) {
  const int w = W >> 2, h = H >> 2;
  const bool ring = r < 2 || r >= H - 2 || c < 2 || c >= W - 2;
  if (!ring) {
    const int i = (r - 2) >> 2, a = (r - 2) & 3, j = (c - 2) >> 2, b = (c - 2) & 3;
    const float wt = (float)wt_of((a + 2) & 3), wl = (float)wl_of((b + 2) & 3);
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
  const int i = (r <= 1) ? 0 : h - 1;  // rows 0/1: line of D row 0; rows H-2/H-1: D row h-1
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

// ========================================================== pass 2, one row
// Output row r (window rows a = r-1, b = r, c = r+1) of this lane.  T / B are
// the D rows above / below for the vertical interpolation; Dc is D row k
// (for the border lines of rows 0,1,H-2,H-1).
template <int kA>  // r - 4k, 0..3
__device__ __forceinline__ void p2_row(const RowD &ra, const RowD &rb, const RowD &rc, const float4 &T,
                                       const float4 &B, const float4 &Dc, int r, int c0, int W, int H,
                                       uint32_t lut_q, uint8_t *orow, bool store) {
  uint32_t pe[4], MX[4], MN[4];
  sobel(ra, rb, rc, pe);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    MX[i] = __vimax3_u16x2(ra.mx[i], rb.mx[i], rc.mx[i]);
    MN[i] = __vimin3_u16x2(ra.mn[i], rb.mn[i], rc.mn[i]);
  }
  // Upscale body (L146, R3): vertical weights (wt, 8-wt) on D rows (T, B),
  // then horizontal; NU = -U, exact.
  constexpr float wt = (float)wt_of(kA), wb = 8.0f - wt;
  const float V0 = __fmaf_rn(wb, B.x, __fmul_rn(wt, T.x));
  const float V1 = __fmaf_rn(wb, B.y, __fmul_rn(wt, T.y));
  const float V2 = __fmaf_rn(wb, B.z, __fmul_rn(wt, T.z));
  const float V3 = __fmaf_rn(wb, B.w, __fmul_rn(wt, T.w));
  constexpr float s = -1.0f / 1024.0f;
  float2 nu01 = lin2(V0, V1, 3 * s, 1 * s, 5 * s, 7 * s);   // x = 0,1: (3,5), (1,7) on (V0, V1)
  float2 nu23 = lin2(V1, V2, 7 * s, 5 * s, 1 * s, 3 * s);   // x = 2,3: (7,1), (5,3) on (V1, V2)
  float2 nu45 = lin2(V1, V2, 3 * s, 1 * s, 5 * s, 7 * s);   // x = 4,5
  float2 nu67 = lin2(V2, V3, 7 * s, 5 * s, 1 * s, 3 * s);   // x = 6,7
  if (r < 2 || r >= H - 2) {  // border rows (warp-uniform): upscale border lines (L140) + frame
    const float q0 = Dc.y, q1 = Dc.z, q2 = Dc.w;  // D row 0 (rows 0,1) or h-1 (rows H-2,H-1)
    nu01 = make_float2(-__fmul_rn(q0, 1.0f / 16.0f), -line_val(q0, q1, 1));
    nu23 = make_float2(-line_val(q0, q1, 2), -line_val(q0, q1, 3));
    nu45 = make_float2(-__fmul_rn(q1, 1.0f / 16.0f), (c0 + 5 == W - 3) ? -__fmul_rn(q1, 1.0f / 16.0f) : -line_val(q1, q2, 1));
    nu67 = make_float2(-line_val(q1, q2, 2), -line_val(q1, q2, 3));
    if (r == 0 || r == H - 1) {  // frame: Sobel 0 (L160), no overshoot window (L208)
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        pe[i] = 0u;
        MX[i] = kF16_255 | (kF16_255 << 16);
        MN[i] = 0u;
      }
    }
  }
  const float NU[8] = {nu01.x, nu01.y, nu23.x, nu23.y, nu45.x, nu45.y, nu67.x, nu67.y};
  float P[8], T8[8], osc[8];
#pragma unroll
  for (int x = 0; x < 8; ++x) {
    const int p = pair_of(x);
    const bool hi = half_of(x);
    const uint32_t qb = __float_as_uint(add_f32_f16(hi ? hi16(pe[p]) : lo16(pe[p]), 8388608.0f));  // 2^23 + pEdge
    const float2 L = lds_f2(qb * 8u + lut_q);                                                      // {adj, osc}
    const float E = add_f32_f16(hi ? hi16(rb.c[p]) : lo16(rb.c[p]), NU[x]);                       // O - U (L148)
    P[x] = __fmaf_rn(L.x, E, -NU[x]);                                                              // L178
    const float mxf = add_f32_f16(hi ? hi16(MX[p]) : lo16(MX[p]), 0.0f);
    const float mnf = add_f32_f16(hi ? hi16(MN[p]) : lo16(MN[p]), 0.0f);
    T8[x] = fminf(fmaxf(P[x], mnf), mxf);  // Fig. 8 branch target (max / min / P)
    osc[x] = L.y;
  }
  uint32_t o[8];
#pragma unroll
  for (int x = 0; x < 8; x += 2) {
    const float2 d = sub2(make_float2(P[x], P[x + 1]), make_float2(T8[x], T8[x + 1]));
    o[x] = cvt_u8(__fmaf_rn(osc[x], d.x, T8[x]));  // osc max / osc min / P, clamp, RNE
    o[x + 1] = cvt_u8(__fmaf_rn(osc[x + 1], d.y, T8[x + 1]));
  }
  if (store) *reinterpret_cast<uint2 *>(orow) = pack8(o);
}

// 12 output rows r0 .. r0+11 (r0 = R0 + 12 m, a multiple of 4); window and D
// rows carried in/out by reference (the unrolled body renames registers).
__device__ __forceinline__ void p2_body12(uint32_t aw, int s0, int lane, RowD &ra, RowD &rb, float4 &Dp, float4 &Dc,
                                          int r0, int c0, int W, int H, uint32_t lut_q, uint8_t *orow, bool active) {
#pragma unroll
  for (int blk = 0; blk < 3; ++blk) {
    const float4 Dn = dblock(aw, s0 + 4 * blk + 4, lane);  // D row k+1 (smem rows of block k+1)
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      const int r = r0 + 4 * blk + a;
      const RowD rc = derive_w<true>(row_words(aw, s0 + 4 * blk + a + 1), lane);
      const bool st = active && r < H;
      uint8_t *op = orow + (size_t)(4 * blk + a) * W;
      if (a == 0) p2_row<0>(ra, rb, rc, Dp, Dc, Dc, r, c0, W, H, lut_q, op, st);
      if (a == 1) p2_row<1>(ra, rb, rc, Dp, Dc, Dc, r, c0, W, H, lut_q, op, st);
      if (a == 2) p2_row<2>(ra, rb, rc, Dc, Dn, Dc, r, c0, W, H, lut_q, op, st);
      if (a == 3) p2_row<3>(ra, rb, rc, Dc, Dn, Dc, r, c0, W, H, lut_q, op, st);
      ra = rb;
      rb = rc;
    }
    Dp = Dc;
    Dc = Dn;
  }
}

__device__ __forceinline__ void p2_warp(uint32_t tile, uint32_t lut, uint8_t *__restrict__ out, int W, int H, int C0w,
                                        int R0, int lane) {
  const int c0 = C0w + 8 * lane;
  const bool active = lane < 30 && c0 < W;
  const uint32_t aw = tile + (uint32_t)(kCol0 + 8 * (lane < 31 ? lane : -1));
  const uint32_t lut_q = lut - (0x4B000000u << 3);  // LDS address of entry p from the bits of (2^23 + p)
  // smem row of global row R0-4 is 0: row r -> r - R0 + 4.
  float4 Dp = dblock(aw, 0, lane);  // D row k0-1
  float4 Dc = dblock(aw, 4, lane);  // D row k0
  RowD ra = derive_w<true>(row_words(aw, 3), lane);
  RowD rb = derive_w<true>(row_words(aw, 4), lane);
  uint8_t *orow = out + (size_t)R0 * W + c0;
  p2_body12(aw, 4, lane, ra, rb, Dp, Dc, R0, c0, W, H, lut_q, orow, active);
  if (R0 + 12 < H)
    p2_body12(aw, 16, lane, ra, rb, Dp, Dc, R0 + 12, c0, W, H, lut_q, orow + (size_t)12 * W, active);

  // Specialised border pass: columns 0,1 and W-2,W-1 inside this tile.
  const bool left = (C0w == 0), right = (C0w <= W - 2 && W - 2 < C0w + kTW);
  if (left || right) {
    __syncwarp();
    const int nr = min(R0 + kTH, H) - R0;
    const int ncol = (left ? 2 : 0) + (right ? 2 : 0);
    for (int idx = lane; idx < nr * ncol; idx += 32) {
      const int r = R0 + idx / ncol;
      const int k = idx % ncol;  // left: columns 0,1; then W-2, W-1
      const int c = left ? (k < 2 ? k : W - 4 + k) : W - 2 + k;
      out[(size_t)r * W + c] = (uint8_t)pixel_generic(tile, lut, r, c, W, H, R0, C0w);
    }
  }
}

// ========================================================== pass 1 (warp)
__device__ __forceinline__ float p1_warp(uint32_t tile, int W, int H, int C0w, int R0, int lane) {
  const int c0 = C0w + 8 * lane;
  const uint32_t aw = tile + (uint32_t)(kCol0 + 8 * (lane < 31 ? lane : -1));
  // Sobel-body pixels of this lane (not frame columns, not beyond the image).
  uint32_t vmask = 0;
#pragma unroll
  for (int x = 0; x < 8; ++x) vmask |= (uint32_t)(c0 + x >= 1 && c0 + x <= W - 2) << x;
  if (lane >= 30) vmask = 0;
  const bool edge = vmask != 0xffu;
  // smem row of global row R0-1 is 0: row r -> r - R0 + 1.
  RowD ra = derive_w<false>(row_words(aw, 0), lane);
  RowD rb = derive_w<false>(row_words(aw, 1), lane);
  float acc = 0.0f;  // exact: < 8 px * 24 rows * 1530 < 2^24
#pragma unroll 1
  for (int m = 0; m < kTH; m += 12) {
#pragma unroll
    for (int a = 0; a < 12; ++a) {
      const int r = R0 + m + a;
      const RowD rc = derive_w<false>(row_words(aw, m + a + 2), lane);
      uint32_t pe[4];
      sobel(ra, rb, rc, pe);
      if (r >= 1 && r < H - 1) {  // Sobel border rows are 0 (L160); rows >= H skipped
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
  }
  return acc;
}

// Last-block-done (sec. V-C stage 2): the frame's mean and lookup tables,
// adj(p) = A (p/m)^gamma and osc(p) = clamp(G exp(-p/(K m)), 0, 1) in f64,
// rounded once to f32 (R9, R11), exactly the oracle's expressions.
__device__ void build_lut(const StepParams &sp, int f) {
  __threadfence();
  const unsigned long long S = atomicAdd(&sp.sums1[f], 0ull);
  const double mean = (double)S / ((double)sp.g.W * (double)sp.g.H);
  const double m = mean > 1.0 ? mean : 1.0;
  for (int p = threadIdx.x; p < kLutSize; p += blockDim.x) {
    float adj = 0.0f, osc = 0.0f;
    if (p <= 1530) {
      adj = (float)((double)sp.prm.amount * pow((double)p / m, (double)sp.prm.gamma));
      osc = (float)fmin(fmax((double)sp.prm.osc_gain * exp(-(double)p / ((double)sp.prm.osc_scale * m)), 0.0), 1.0);
    }
    sp.luts1[(size_t)f * kLutSize + p] = make_float2(adj, osc);
  }
  if (threadIdx.x == 0) {
    sp.means1[f] = mean;
    sp.counters1[f] = 0u;  // re-arm for the next launch
  }
}

__global__ void __launch_bounds__(kThreadsT, 2)
    step_kernel(const __grid_constant__ CUtensorMap map1, const __grid_constant__ CUtensorMap map2, StepParams sp) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint32_t warp_sum[kWarpsT];
  __shared__ int next_task[2];
  __shared__ int last_frame;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar0 = sbase + 2 * kStage;
  const int ntasks = sp.n1 + sp.n2;
  const Geo &g = sp.g;

  if (threadIdx.x == 0) {
    mbar_init(bar0, 1);
    mbar_init(bar0 + 8, 1);
    fence_barrier_init();
  }
  // Producer: grab the next task and start its loads into stage b.
  auto issue = [&](int b) {
    const int t = (int)atomicAdd(sp.task_counter, 1u);
    next_task[b] = t;
    if (t >= ntasks) return;
    const bool p1 = t < sp.n1;
    int f, C0, R0;
    tile_of(g, p1 ? t : t - sp.n1, f, C0, R0);
    int nw = 0;
#pragma unroll
    for (int w = 0; w < kWarpsT; ++w) nw += (C0 + w * kTW < g.W);
    const uint32_t bar = bar0 + 8u * b, st = sbase + (uint32_t)(b * kStage);
    fence_proxy_async();
    if (p1) {
      mbar_expect_tx(bar, (uint32_t)(nw * kBox1));
      for (int w = 0; w < nw; ++w) tma_box(st + w * kSlot, &map1, C0 + w * kTW, R0 - 1, f, bar);
    } else {
      mbar_expect_tx(bar, (uint32_t)(nw * kBox2 + kLutBytes));
      for (int w = 0; w < nw; ++w) tma_box(st + w * kSlot, &map2, C0 + w * kTW, R0 - 4, f, bar);
      bulk_copy(st + kWarpsT * kSlot, sp.luts2 + (size_t)f * kLutSize, kLutBytes, bar);
    }
  };
  if (threadIdx.x == 0) issue(0);
  __syncthreads();

  for (int i = 0;; ++i) {
    const int b = i & 1;
    const int t = next_task[b];
    if (t >= ntasks) break;
    if (threadIdx.x == 0) issue(b ^ 1);  // stage b^1 was released by the barrier ending iteration i-1
    mbar_wait(bar0 + 8u * b, (uint32_t)((i >> 1) & 1));
    const uint32_t st = sbase + (uint32_t)(b * kStage);
    const bool p1 = t < sp.n1;
    int f, C0, R0;
    tile_of(g, p1 ? t : t - sp.n1, f, C0, R0);
    const int C0w = C0 + warp * kTW;
    if (!p1) {
      if (C0w < g.W)
        p2_warp(st + warp * kSlot, st + kWarpsT * kSlot, sp.out2 + (size_t)f * g.W * g.H, g.W, g.H, C0w, R0, lane);
    } else {
      const float acc = (C0w < g.W) ? p1_warp(st + warp * kSlot, g.W, g.H, C0w, R0, lane) : 0.0f;
      const uint32_t ws = __reduce_add_sync(0xffffffffu, (uint32_t)acc);
      if (lane == 0) warp_sum[warp] = ws;
      __syncthreads();
      if (threadIdx.x == 0) {
        unsigned long long part = 0;
#pragma unroll
        for (int w = 0; w < kWarpsT; ++w) part += warp_sum[w];
        atomicAdd(&sp.sums1[f], part);
        __threadfence();
        const unsigned int ticket = atomicAdd(&sp.counters1[f], 1u);
        last_frame = (ticket == (unsigned)g.per_frame - 1) ? f : -1;
      }
      __syncthreads();
      if (last_frame >= 0) build_lut(sp, last_frame);
    }
    __syncthreads();  // stage b is free again
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
  const cuuint64_t dims[4] = {16, (cuuint64_t)W / 16, (cuuint64_t)H, (cuuint64_t)n};  // [n][H][W/16][16]
  const cuuint64_t strides[3] = {16, (cuuint64_t)W, (cuuint64_t)W * H};
  const cuuint32_t box[4] = {16, (cuuint32_t)kChunks, (cuuint32_t)box_rows, 1};
  const cuuint32_t estr[4] = {1, 1, 1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, (void *)imgs, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
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

int tma_tasks(int n, int W, int H) {
  const int tx = (W + kCtaCols - 1) / kCtaCols, ty = (H + kTH - 1) / kTH;
  return tx * ty * n;
}

cudaError_t launch_step_tma(const StepLaunch &a, int W, int H, const Params &p, cudaStream_t stream) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(step_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem);
    attr = true;
  }
  CUtensorMap m1, m2;
  memset(&m1, 0, sizeof(m1));
  memset(&m2, 0, sizeof(m2));
  if (a.n1 > 0 && !make_map(&m1, a.in1, a.n1, W, H, kRows1)) return cudaErrorInvalidValue;
  if (a.n2 > 0 && !make_map(&m2, a.in2, a.n2, W, H, kRows2)) return cudaErrorInvalidValue;
  StepParams sp;
  sp.g.W = W;
  sp.g.H = H;
  sp.g.tiles_x = (W + kCtaCols - 1) / kCtaCols;
  sp.g.per_frame = sp.g.tiles_x * ((H + kTH - 1) / kTH);
  sp.n1 = a.n1 * sp.g.per_frame;
  sp.n2 = a.n2 * sp.g.per_frame;
  sp.prm = p;
  sp.sums1 = a.sums1;
  sp.means1 = a.means1;
  sp.counters1 = a.counters1;
  sp.luts1 = a.luts1;
  sp.luts2 = a.luts2;
  sp.out2 = a.out2;
  sp.task_counter = a.task_counter;
  const int tasks = sp.n1 + sp.n2;
  if (tasks == 0) return cudaSuccess;
  const int grid = std::min(tasks, 2 * num_sms());
  step_kernel<<<grid, kThreadsT, kSmem, stream>>>(m1, m2, sp);
  return cudaGetLastError();
}

}  // namespace sharp
