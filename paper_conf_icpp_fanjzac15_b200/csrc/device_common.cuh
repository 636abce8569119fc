// Device helpers shared by the sm_100a kernels (kernels.cu: generic LDG
// path; kernels_tma.cu: TMA-staged persistent path).  Nothing here is shared
// with the CPU oracle.
#pragma once
#include <cuda_fp16.h>
#include <stdint.h>

#include "kernels.h"

namespace sharp {
namespace dev {

// ------------------------------------------------------------------ bit/f16
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t s) { return __byte_perm(a, b, s); }
__device__ __forceinline__ __half2 H(uint32_t u) {
  __half2 h;
  *reinterpret_cast<uint32_t *>(&h) = u;
  return h;
}
__device__ __forceinline__ uint32_t U32(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }
__device__ __forceinline__ uint32_t hadd(uint32_t a, uint32_t b) { return U32(__hadd2(H(a), H(b))); }
__device__ __forceinline__ uint32_t hsub(uint32_t a, uint32_t b) { return U32(__hsub2(H(a), H(b))); }
__device__ __forceinline__ uint32_t hfma(uint32_t a, uint32_t b, uint32_t c) {
  return U32(__hfma2(H(a), H(b), H(c)));
}
__device__ __forceinline__ uint32_t habsadd(uint32_t a, uint32_t b) {
  return U32(__hadd2(__habs2(H(a)), __habs2(H(b))));
}
// f32 + f16 (sm_100 mixed-precision add, one FHADD); exact for the values used.
__device__ __forceinline__ float add_f32_f16(uint16_t a, float c) {
  float d;
  asm("add.f32.f16 %0, %1, %2;" : "=f"(d) : "h"(a), "f"(c));
  return d;
}
// f16 * f16 + f32 (sm_100 mixed-precision FMA, one FHFMA); exact for the values used.
__device__ __forceinline__ float fma_f32_f16(uint16_t a, uint16_t b, float c) {
  float d;
  asm("fma.rn.f32.f16 %0, %1, %2, %3;" : "=f"(d) : "h"(a), "h"(b), "f"(c));
  return d;
}
__device__ __forceinline__ uint16_t lo16(uint32_t u) { return (uint16_t)(u & 0xffffu); }
__device__ __forceinline__ uint16_t hi16(uint32_t u) { return (uint16_t)(u >> 16); }
// Round half to even and saturate to [0, 255] (R14 + the final clamp of Fig. 8).
__device__ __forceinline__ uint32_t cvt_u8(float a) {
  uint32_t r;
  asm("cvt.rni.sat.u8.f32 %0, %1;" : "=r"(r) : "f"(a));
  return r;
}
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float2 lds_f2(uint32_t addr) {
  float2 v;
  asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t addr) {
  uint32_t v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint2 lds_u64(uint32_t addr) {
  uint2 v;
  asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t addr) {
  uint16_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(addr));
  return v;
}

constexpr uint32_t kF16Bias = 0x64646464u;    // byte 0x64 -> f16 exponent of 1024
constexpr uint32_t kMinus1024 = 0xE400E400u;  // (-1024, -1024) as f16x2
constexpr uint32_t kTwo = 0x40004000u;        // (2, 2)
constexpr uint32_t kF16_255 = 0x5BF8u;        // 255.0 as f16

// A row of a lane's 8 pixels plus one halo column each side, as words:
// pw = columns c0-4..c0-1, w0 = c0..c0+3, w1 = c0+4..c0+7, nw = c0+8..c0+11.
struct Words {
  uint32_t pw, w0, w1, nw;
};

// Pair layout (f16x2, low half first):
//   p[0] = (c0, c0+2)   p[1] = (c0+1, c0+3)   p[2] = (c0+4, c0+6)   p[3] = (c0+5, c0+7)
__host__ __device__ constexpr int pair_of(int x) { return (x & 1) + ((x >> 2) << 1); }
__host__ __device__ constexpr int half_of(int x) { return (x >> 1) & 1; }

// Per image row: what the 3-row window needs (all f16x2, exact integers).
struct RowD {
  uint32_t h[4];   // right - left neighbour (Gx ingredient)
  uint32_t s[4];   // left + 2 centre + right (Gy ingredient)
  uint32_t mx[4];  // max of left/centre/right (u16 order of non-negative f16 == value order)
  uint32_t mn[4];
  uint32_t c[4];   // centre values
};

template <bool kMinMax>
__device__ __forceinline__ RowD derive(const Words &x) {
  const uint32_t E0 = hadd(prmt(x.w0, kF16Bias, 0x4240), kMinus1024);  // (c0, c0+2)
  const uint32_t O0 = hadd(prmt(x.w0, kF16Bias, 0x4341), kMinus1024);  // (c0+1, c0+3)
  const uint32_t E1 = hadd(prmt(x.w1, kF16Bias, 0x4240), kMinus1024);  // (c0+4, c0+6)
  const uint32_t O1 = hadd(prmt(x.w1, kF16Bias, 0x4341), kMinus1024);  // (c0+5, c0+7)
  const uint32_t PO = hadd(prmt(x.pw, kF16Bias, 0x4341), kMinus1024);  // (c0-3, c0-1)
  const uint32_t NE = hadd(prmt(x.nw, kF16Bias, 0x4240), kMinus1024);  // (c0+8, c0+10)
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

// pEdge of the middle row b (L166: |Gx| + |Gy| of the standard Sobel pair, R7).
__device__ __forceinline__ void sobel(const RowD &a, const RowD &b, const RowD &c, uint32_t pe[4]) {
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t gx = hadd(hfma(kTwo, b.h[i], a.h[i]), c.h[i]);
    const uint32_t gy = hsub(c.s[i], a.s[i]);
    pe[i] = habsadd(gx, gy);
  }
}

// Overwrite the f16 lane of pixel x with `fill`.
__device__ __forceinline__ void set_px(uint32_t v[4], int x, uint32_t fill) {
#pragma unroll
  for (int i = 0; i < 8; ++i)
    if (i == x) {
      const int p = pair_of(i);
      v[p] = half_of(i) ? ((v[p] & 0xffffu) | (fill << 16)) : ((v[p] & 0xffff0000u) | fill);
    }
}

// Sum of a 4x4 block of bytes given as 4 words (16 * D, exact).
__device__ __forceinline__ uint32_t blk4(uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  uint32_t s = __dp4a(a, 0x01010101u, 0u);
  s = __dp4a(b, 0x01010101u, s);
  s = __dp4a(c, 0x01010101u, s);
  return __dp4a(d, 0x01010101u, s);
}

// Upscale body weights (R3): P = [[7,1],[5,3],[3,5],[1,7]] / 8.  For lane
// column x (0..7) of an 8-aligned group at c0 (D column j0 = c0/4): the left D
// column relative to j0-1 (0..2) and the left weight (times 8).
__host__ __device__ constexpr int jl_of(int x) { return x < 2 ? 0 : (x < 6 ? 1 : 2); }
__host__ __device__ constexpr int wl_of(int x) {
  return (x & 3) == 0 ? 3 : (x & 3) == 1 ? 1 : (x & 3) == 2 ? 7 : 5;
}
// Vertical weight of the top D row for row offset a' = r - 4k (0..3).
__host__ __device__ constexpr int wt_of(int a) { return a == 0 ? 3 : a == 1 ? 1 : a == 2 ? 7 : 5; }

// line(v, n)[c] of L140 from 16*D values x = v[c>>2], y = v[(c>>2)+1] and
// k = c & 3: ((4-k) x + k y) / 4, as U (/16): exact.
__device__ __forceinline__ float line_val(float x16, float y16, int k) {
  return __fmul_rn(__fadd_rn(__fmul_rn((float)(4 - k), x16), __fmul_rn((float)k, y16)), 1.0f / 64.0f);
}

// ------------------------------------------------------- upscale border (R4, R5)
// Final value of U at a pixel of the 2-pixel ring (last writer of steps
// i..vii of L140-L142).  Sc = 16*D of the current D row block (row k) for
// columns j0-1..j0+2, Sn = the next D row (k+1); j0 = c0/4; r = 4k + a'.
// col_wins: the R5 alternative (column work after the row work: the top-left
// 2x2 keeps the column line's values instead of D[0][0]).
__device__ __forceinline__ float ring_u(int r, int c, int W, int H, int j0, const float (&Sc)[4], const float (&Sn)[4],
                                        bool col_wins) {
  const int w = W >> 2, h = H >> 2;
  auto col = [&](int j) { return j - j0 + 1; };  // index into Sc/Sn (0..3)
  // register selects instead of a dynamically indexed local array (no stack frame)
  auto at = [](const float(&a)[4], int i) { return i <= 0 ? a[0] : i == 1 ? a[1] : i == 2 ? a[2] : a[3]; };
  if (r >= H - 2 && c >= W - 2) {                 // (vii): third last of last column = D[h-1][w-1]
    return __fmul_rn(at(Sc, col(w - 1)), 1.0f / 16.0f);
  }
  if ((c <= 1 || c >= W - 2) && r <= H - 3) {     // (vi)/(ii)/(iv): column lines
    const int j = (c <= 1) ? 0 : w - 1;
    if (c <= 1 && r <= 1 && !col_wins) return __fmul_rn(at(Sc, col(0)), 1.0f / 16.0f);  // (v) then (vi): D[0][0]
    const int rr = (r == H - 3) ? H - 4 : r;   // third last <- fourth last
    const int k = rr & 3;                      // rr>>2 == current D row (rr in the block of r)
    return line_val(at(Sc, col(j)), at(Sn, col(j)), k);
  }
  // rows 0/1 (line of D row 0) or H-2/H-1 (line of D row h-1); Sc is that D row.
  const int cc = (c == W - 3) ? W - 4 : c;
  const int jj = cc >> 2, k = cc & 3;
  const float x = at(Sc, col(jj));
  const float y = (k == 0) ? x : at(Sc, col(jj + 1));
  (void)h;
  return line_val(x, y, k);
}

// Preliminary (L178) and overshoot (Fig. 8) for one pixel:
//   P = fma(adj, E, U);  t = clamp(P, mn, mx)  (== the branch target of
//   Fig. 8: max if P > max, min if P < min, else P);  F = fma(osc, P - t, t)
//   (osc max / osc min / P);  out = RNE(clamp(F, 0, 255)).
// Bit-identical to the oracle's branchy form.
__device__ __forceinline__ uint32_t sharpen_px(float adj, float osc, float E, float U, float mxf, float mnf) {
  const float P = __fmaf_rn(adj, E, U);
  const float t = fminf(fmaxf(P, mnf), mxf);
  const float F = __fmaf_rn(osc, __fsub_rn(P, t), t);
  return cvt_u8(F);
}

// Round half to even, saturate to [0, 255] and pack four values into one
// word (bytes a, b, c, d from low to high).  cvt.rni.s32 + cvt.pack.sat.u8
// is the same function as cvt.rni.sat.u8.f32 (R14); ptxas fuses each pair
// into one two-source F2IP.U8 (4 pixels in 2 instructions instead of 4 F2IP
// + 3 PRMT).
__device__ __forceinline__ uint32_t pack4_rni_u8(float a, float b, float c, float d) {
  uint32_t r;
  asm("{\n"
      ".reg .b32 t0, t1, t2, t3, lo;\n"
      "cvt.rni.s32.f32 t2, %3;\n"
      "cvt.rni.s32.f32 t3, %4;\n"
      "cvt.pack.sat.u8.s32.b32 lo, t3, t2, 0;\n"
      "cvt.rni.s32.f32 t0, %1;\n"
      "cvt.rni.s32.f32 t1, %2;\n"
      "cvt.pack.sat.u8.s32.b32 %0, t1, t0, lo;\n"
      "}"
      : "=r"(r)
      : "f"(a), "f"(b), "f"(c), "f"(d));
  return r;
}

// Truncate toward zero and saturate to [0, 255] (the R14 alternative).
__device__ __forceinline__ uint32_t cvt_u8_rz(float a) {
  uint32_t r;
  asm("cvt.rzi.sat.u8.f32 %0, %1;" : "=r"(r) : "f"(a));
  return r;
}

// ---------------------------------------------------------- per-frame tables
// L174: the mean of pEdge over the W*H elements (R8), or over the (W-2)(H-2)
// body (the R8 alternative); S is exact.
__device__ __forceinline__ double frame_mean(unsigned long long S, int W, int H, int flags) {
  return (flags & kReadInteriorMean) ? (double)S / ((double)(W - 2) * (double)(H - 2))
                                     : (double)S / ((double)W * (double)H);
}
// {adj(p), osc(p)} for pEdge value p (f64, rounded once to f32; R9, R11, R15):
//   adj = A (p / m)^gamma        (R9)   or A (1 - exp(-p / (K m)))   (R9 alternative)
//   osc = clamp(G exp(-p / (K m)), 0, 1)   (R11)   or G               (R11 alternative)
// with m = max(mean, 1).
__device__ __forceinline__ float lut_adj(int p, double mean, const Params &prm) {
  const double m = mean > 1.0 ? mean : 1.0;
  return (prm.flags & kReadStrengthExp)
             ? (float)((double)prm.amount * (1.0 - exp(-(double)p / ((double)prm.osc_scale * m))))
             : (float)((double)prm.amount * pow((double)p / m, (double)prm.gamma));
}
__device__ __forceinline__ float lut_osc(int p, double mean, const Params &prm) {
  const double m = mean > 1.0 ? mean : 1.0;
  return (prm.flags & kReadOscConst)
             ? prm.osc_gain
             : (float)fmin(fmax((double)prm.osc_gain * exp(-(double)p / ((double)prm.osc_scale * m)), 0.0), 1.0);
}
__device__ __forceinline__ float2 lut_entry(int p, double mean, const Params &prm) {
  return make_float2(lut_adj(p, mean, prm), lut_osc(p, mean, prm));
}

// The same with truncation (the R14 alternative): cvt.rzi then the saturating pack.
__device__ __forceinline__ uint32_t pack4_rzi_u8(float a, float b, float c, float d) {
  uint32_t r;
  asm("{\n"
      ".reg .b32 t0, t1, t2, t3, lo;\n"
      "cvt.rzi.s32.f32 t2, %3;\n"
      "cvt.rzi.s32.f32 t3, %4;\n"
      "cvt.pack.sat.u8.s32.b32 lo, t3, t2, 0;\n"
      "cvt.rzi.s32.f32 t0, %1;\n"
      "cvt.rzi.s32.f32 t1, %2;\n"
      "cvt.pack.sat.u8.s32.b32 %0, t1, t0, lo;\n"
      "}"
      : "=r"(r)
      : "f"(a), "f"(b), "f"(c), "f"(d));
  return r;
}

// Packs 8 bytes (low byte of each word) into two words.
__device__ __forceinline__ uint2 pack8(const uint32_t o[8]) {
  const uint32_t a = prmt(prmt(o[0], o[1], 0x0040), prmt(o[2], o[3], 0x0040), 0x5410);
  const uint32_t b = prmt(prmt(o[4], o[5], 0x0040), prmt(o[6], o[7], 0x0040), 0x5410);
  return make_uint2(a, b);
}

}  // namespace dev
}  // namespace sharp
