// Device pieces shared by the TMA-staged sm_100a kernels (kernels_tma.cu:
// the step kernel; kernels_res.cu: the TMEM-resident kernel): the CTA /
// warp tile geometry, TMA + mbarrier wrappers, L2 policies, packed f32x2
// helpers, the smem row window (lane words, f16x2 derivation, D block sums)
// and the 2-pixel ring overrides.  Internal to libsharp; nothing here is
// shared with the CPU oracle.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "device_common.cuh"
#include "kernels.h"

namespace sharp {
namespace {
using namespace dev;

constexpr int kTW = 240;     // output columns per warp tile (lanes 0..29 x 8 px)
constexpr int kTH = 12;      // output rows per (pass-2) warp tile
constexpr int kWarpsT = 4;   // compute warps = warp tiles per CTA tile
constexpr int kCtaCols = kTW * kWarpsT;
constexpr int kThreadsT = 32 * (kWarpsT + 1);  // + producer warp
// pEdge = |Gx| + |Gy| is always even (Gx and Gy both have the parity of the
// sum of the four window corners), so the TMA kernels' tables hold the even
// entries only: entry k = pEdge / 2, k < kLut2 (766 used).
constexpr int kLut2 = 768;
constexpr int kLutBytes = kLut2 * 8;
constexpr unsigned kPollNs = 100;  // dependency polling interval of the producer
// A warp tile needs columns C0w-8 .. C0w+247.  TMA box starts must be
// 16-byte aligned in the innermost dimension and a box dimension is at most
// 256, so a warp tile is fetched as one 256-column box of the [n][H][W]
// frames (region A, smem pitch 256).  The step kernel (kernels_tma.cu) loads
// C0w-16 .. C0w+239 for warps 0..2 and C0w .. C0w+255 for the last warp, so
// every halo lies in some warp's region A; the resident kernel
// (kernels_res.cu) keeps a 16-column region B (pitch 16) for the last warp's
// right halo.  (When the next warp has no columns, the halo lies beyond the
// image and only feeds pixels that are either not stored or on the
// overridden frame column W-1.)
constexpr int kPitch = 256;           // region A pitch
constexpr int kPitchB = 16;           // region B pitch
constexpr int kCol0 = 16;             // region-A column of C0w
constexpr int kRows2 = kTH + 8;       // pass-2 box rows: R0-4 .. R0+kTH+3
constexpr int kSlot = kPitch * kRows2;  // per-warp smem slot: region A (128-B aligned)
static_assert(kSlot % 128 == 0, "TMA smem destinations must be 128-B aligned");
static_assert(kTH % 3 == 0 && kTH % 4 == 0, "row loop is unrolled by 3, D blocks are 4 rows");
static_assert(kLut2 <= kLutSize && 2 * (kLut2 - 1) >= 1530, "even-pEdge tables");

// ------------------------------------------------------------ TMA / mbarrier
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, 1000000;\n"  // suspend (not spin) up to 1 ms
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
// Waits with test_wait polls and an exponential nanosleep back-off (64 ns ..
// max_ns): a waiting warp issues a few instructions per microsecond instead
// of spinning on try_wait, whose suspend wakes on any barrier event.
__device__ __forceinline__ bool mbar_test_one(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_backoff(uint32_t bar, uint32_t parity, unsigned max_ns) {
  unsigned ns = 64;
  while (!mbar_test_one(bar, parity)) {
    __nanosleep(ns);
    ns = ns < max_ns ? 2 * ns : max_ns;
  }
}
// One 3-D box {cols, rows, 1} of the [n][H][W] frames at (x, r, f) (x 16-B aligned).
// L2 eviction-priority policies (createpolicy): pass-1 loads keep the frame
// in L2 for its pass-2 re-read (evict_last); pass-2 loads and the output
// stores are the last touch (evict_first).
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void tma_box(uint32_t dst, const CUtensorMap *map, int x, int r, int f, uint32_t bar,
                                        uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, "
      "{%2, %3, %4}], [%5], %6;" ::"r"(dst),
      "l"(map), "r"(x), "r"(r), "r"(f), "r"(bar), "l"(policy)
      : "memory");
}
// Output store.  (Measured: an L2::cache_hint store costs ~5% of the step
// through extra issue; plain STG.64 it is.)
__device__ __forceinline__ void st_stream_u64(uint8_t *p, uint2 v, uint64_t policy) {
  (void)policy;
  *reinterpret_cast<uint2 *>(p) = v;
}
__device__ __forceinline__ void bulk_copy(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void fence_barrier_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ unsigned int ld_acquire(const unsigned int *p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
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
// (a*x + b*y) for a lane pair with the same (x, y): FMUL2 then FFMA2, each
// single-rounding per lane -- bit-identical to the scalar fmul/fma pair.
__device__ __forceinline__ float2 lin2(float x, float y, unsigned long long a, unsigned long long b) {
  unsigned long long t, r;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(t) : "l"(f2pack(x, x)), "l"(a));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(f2pack(y, y)), "l"(b), "l"(t));
  return f2unpack(r);
}
__device__ __forceinline__ float2 sub2(float2 a, float2 b) {
  unsigned long long r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(f2pack(a.x, a.y)), "l"(f2pack(b.x, b.y)));
  return f2unpack(r);
}

// Polling loads: relaxed (no L1 invalidation per poll); the caller issues
// one acquire fence after the awaited value was seen.
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned int ld_relaxed_u32(const unsigned int *p) {
  unsigned int v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acquire() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
// Peer-memory all-reduce inside the launch (kStepBandFused): system-scope
// release stores into the other bands' windows, acquire polls of our own.
__device__ __forceinline__ void st_release_sys_u64(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys_u64(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long gtime_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// ------------------------------------------------------------- row window
// A lane's row window in a stage: its 8 bytes of smem row s at base + s * pitch.
struct LaneRow {
  uint32_t base, pitch;
};
__device__ __forceinline__ uint2 row_words(const LaneRow &a, int s) { return lds_u64(a.base + (uint32_t)s * a.pitch); }

// Converts a row of words into the window data.  Neighbour pairs come from
// the adjacent lanes (shuffle), so each lane loads only its own 8 bytes.
// kDenorm (pass 1 of the step kernel, which only sums pEdge): the bytes
// become the f16 SUBNORMALS b * 2^-24 (one PRMT with zero bytes, no HADD2);
// f16 arithmetic keeps subnormals and every integer k * 2^-24 with |k| <=
// 2048 is exact, so the Sobel values are pEdge * 2^-24 exactly.
template <bool kMinMax, bool kDenorm = false>
__device__ __forceinline__ RowD derive_w(uint2 w, int lane) {
  auto unpack = [](uint32_t x, uint32_t sel) {
    return kDenorm ? prmt(x, 0u, sel) : hadd(prmt(x, kF16Bias, sel), kMinus1024);
  };
  const uint32_t E0 = unpack(w.x, 0x4240);  // (c0, c0+2)
  const uint32_t O0 = unpack(w.x, 0x4341);  // (c0+1, c0+3)
  const uint32_t E1 = unpack(w.y, 0x4240);  // (c0+4, c0+6)
  const uint32_t O1 = unpack(w.y, 0x4341);  // (c0+5, c0+7)
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
    if (kDenorm) {
      // s = l + 2c + r <= 1020 units: non-negative and < 2048, so its f16
      // bit pattern is the integer itself -- two u16 lanes of plain integer
      // adds (no carry between the halves: bytes < 2^8) instead of f16
      // FMA-pipe ops (measured +1.4% on the 1024-frame step: pass 1 was
      // throttled on the FMA pipe).
      uint32_t t;
      asm("add.u32 %0, %1, %2;" : "=r"(t) : "r"(l[i]), "r"(p[i]));
      asm("add.u32 %0, %1, %2;" : "=r"(t) : "r"(t), "r"(p[i]));
      asm("add.u32 %0, %1, %2;" : "=r"(d.s[i]) : "r"(t), "r"(r[i]));
    } else {
      d.s[i] = hadd(hfma(kTwo, p[i], l[i]), r[i]);
    }
    if (kMinMax) {
      d.mx[i] = __vimax3_u16x2(l[i], p[i], r[i]);
      d.mn[i] = __vimin3_u16x2(l[i], p[i], r[i]);
    }
  }
  return d;
}

// D sums (16*D) of the block at smem rows s..s+3 for D columns j0-1..j0+2.
__device__ __forceinline__ float4 dblock(const LaneRow &a, int s, int lane) {
  const uint32_t o = a.base + (uint32_t)s * a.pitch;
  const uint2 r0 = lds_u64(o), r1 = lds_u64(o + a.pitch), r2 = lds_u64(o + 2 * a.pitch), r3 = lds_u64(o + 3 * a.pitch);
  const float d0 = (float)blk4(r0.x, r1.x, r2.x, r3.x);
  const float d1 = (float)blk4(r0.y, r1.y, r2.y, r3.y);
  const float dm1 = __shfl_sync(0xffffffffu, d1, (lane + 31) & 31);
  const float d2 = __shfl_sync(0xffffffffu, d0, (lane + 1) & 31);
  return make_float4(dm1, d0, d1, d2);
}

// ========================================================== pass 2, one row (pieces)
// Packed horizontal weights -w/1024 for pixel pairs (x, x+1), in the constant
// bank (loaded with LDC where used; as literals, ptxas kept rematerialising
// them on every row under the 128-register cap -- measured 4% slower).
// {lo, hi} = {-3, -1}, {-5, -7}, {-7, -5}, {-1, -3} / 1024 as f32 bit pairs.
__constant__ unsigned long long c_wts[4] = {0xba800000bb400000ull, 0xbbe00000bba00000ull, 0xbba00000bbe00000ull,
                                            0xbb400000ba800000ull};
__device__ __forceinline__ unsigned long long cwt(int i) { return c_wts[i]; }
__device__ __forceinline__ float div16(float s) { return __fmul_rn(s, 1.0f / 16.0f); }

// The 2-pixel ring (L140-L142 upscale border, L160 Sobel frame, L208
// overshoot frame): overrides of -U, pEdge and the overshoot window.
__device__ __forceinline__ void set_frame_px(uint32_t pe[4], uint32_t MX[4], uint32_t MN[4], int x) {
  set_px(pe, x, 0u);         // Sobel frame: 0
  set_px(MX, x, kF16_255);   // overshoot frame: the clamped preliminary value,
  set_px(MN, x, 0u);         // i.e. window [0, 255]
}
// The frame columns 0 / W-1 of the edge lanes (L160, L208): pEdge 0, window
// [0, 255]; column 0 is the low half of pair 0, W-1 the high half of pair 3.
// Selects, not branches: no lane-divergent control flow in the row loop.
__device__ __forceinline__ void frame_cols(uint32_t pe[4], uint32_t MX[4], uint32_t MN[4], int edge) {
  const bool e1 = edge == 1, e2 = edge == 2;
  const uint32_t k0 = e1 ? 0xffff0000u : 0xffffffffu, k3 = e2 ? 0x0000ffffu : 0xffffffffu;
  pe[0] &= k0;
  MN[0] &= k0;
  MX[0] = (MX[0] & k0) | (e1 ? kF16_255 : 0u);
  pe[3] &= k3;
  MN[3] &= k3;
  MX[3] = (MX[3] & k3) | (e2 ? (kF16_255 << 16) : 0u);
}
// Columns 0,1 / W-2,W-1 on rows 2..H-3 with the column line's value given:
// v = -U of this row (the step kernel keeps it incrementally).
__device__ __forceinline__ void ring_cols_v(float NU[8], uint32_t pe[4], uint32_t MX[4], uint32_t MN[4], float v,
                                            int edge) {
  const bool e1 = edge == 1, e2 = edge == 2;
  NU[0] = e1 ? v : NU[0];
  NU[1] = e1 ? v : NU[1];
  NU[6] = e2 ? v : NU[6];
  NU[7] = e2 ? v : NU[7];
  frame_cols(pe, MX, MN, edge);
}
// Rows 0,1 (line of D row 0) and H-2,H-1 (line of D row h-1): here D0 is
// that D row; the corners follow the step order (v)-(vii).
__device__ __forceinline__ void ring_rows(float NU[8], uint32_t pe[4], uint32_t MX[4], uint32_t MN[4],
                                          const float4 &D0, const float4 &D1, int r, int c0, int W, int H,
                                          int edge) {
  const float q0 = D0.y, q1 = D0.z, q2 = D0.w;
  float u[8] = {div16(q0),         line_val(q0, q1, 1), line_val(q0, q1, 2), line_val(q0, q1, 3),
                div16(q1),         line_val(q1, q2, 1), line_val(q1, q2, 2), line_val(q1, q2, 3)};
  // (lane-dependent choices as selects: no divergent control flow in the row loop)
  u[5] = (c0 + 5 == W - 3) ? div16(q1) : u[5];  // third last <- fourth last
  const bool top = r < 2;
  u[1] = (edge == 1 && top) ? div16(q0) : u[1];  // (v)+(vi): top-left 2x2 = D[0][0]
  // columns W-2, W-1 (D column w-1 = j0+1)
  const float v = (top && r == 1) ? line_val(D0.z, D1.z, 1) : div16(D0.z);
  u[6] = edge == 2 ? v : u[6];
  u[7] = edge == 2 ? v : u[7];
#pragma unroll
  for (int x = 0; x < 8; ++x) NU[x] = -u[x];
  frame_cols(pe, MX, MN, edge);  // column 0 / W-1 (rows 1, H-2)
  if (r == 0 || r == H - 1) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      pe[i] = 0u;
      MX[i] = kF16_255 | (kF16_255 << 16);
      MN[i] = 0u;
    }
  }
}
// Columns 0,1 / W-2,W-1 on rows 2..H-3 (lines of D columns 0 / w-1).
__device__ __forceinline__ void ring_cols(float NU[8], uint32_t pe[4], uint32_t MX[4], uint32_t MN[4],
                                          const float4 &D0, const float4 &D1, int r, int H, int edge) {
  const int rr = (r == H - 3) ? H - 4 : r;  // third last <- fourth last
  const int k = rr & 3;
  const float x0 = edge == 1 ? D0.y : D0.z, x1 = edge == 1 ? D1.y : D1.z;
  const float v = -(k == 0 ? div16(x0) : line_val(x0, x1, k));
  if (edge == 1) {
    NU[0] = v;
    NU[1] = v;
    set_frame_px(pe, MX, MN, 0);
  } else if (edge == 2) {
    NU[6] = v;
    NU[7] = v;
    set_frame_px(pe, MX, MN, 7);
  }
}

#ifndef SHARP_F4_PACKED
#define SHARP_F4_PACKED 1
#endif
__device__ __forceinline__ float4 f4fma(float a, const float4 &x, const float4 &y) {  // a*x + y, exact here
  if (SHARP_F4_PACKED) {  // two packed f32x2 FMAs (single rounding per lane, as the scalar form)
    unsigned long long lo, hi;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(lo) : "l"(f2pack(a, a)), "l"(f2pack(x.x, x.y)), "l"(f2pack(y.x, y.y)));
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(hi) : "l"(f2pack(a, a)), "l"(f2pack(x.z, x.w)), "l"(f2pack(y.z, y.w)));
    const float2 l = f2unpack(lo), h = f2unpack(hi);
    return make_float4(l.x, l.y, h.x, h.y);
  }
  return make_float4(__fmaf_rn(a, x.x, y.x), __fmaf_rn(a, x.y, y.y), __fmaf_rn(a, x.z, y.z), __fmaf_rn(a, x.w, y.w));
}
__device__ __forceinline__ float4 f4add(const float4 &x, const float4 &y) {  // two packed f32x2 adds
  unsigned long long lo, hi;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(lo) : "l"(f2pack(x.x, x.y)), "l"(f2pack(y.x, y.y)));
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(hi) : "l"(f2pack(x.z, x.w)), "l"(f2pack(y.z, y.w)));
  const float2 a = f2unpack(lo), b = f2unpack(hi);
  return make_float4(a.x, a.y, b.x, b.y);
}
__device__ __forceinline__ float4 f4twice_diff(const float4 &x, const float4 &y) {  // 2 (x - y), exact here
  if (SHARP_F4_PACKED) {  // packed sub then packed mul (exact: integers < 2^13)
    unsigned long long lo, hi;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(lo) : "l"(f2pack(x.x, x.y)), "l"(f2pack(y.x, y.y)));
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(hi) : "l"(f2pack(x.z, x.w)), "l"(f2pack(y.z, y.w)));
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(lo) : "l"(lo), "l"(f2pack(2.0f, 2.0f)));
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(hi) : "l"(hi), "l"(f2pack(2.0f, 2.0f)));
    const float2 l = f2unpack(lo), h = f2unpack(hi);
    return make_float4(l.x, l.y, h.x, h.y);
  }
  return make_float4(__fmul_rn(2.0f, __fsub_rn(x.x, y.x)), __fmul_rn(2.0f, __fsub_rn(x.y, y.y)),
                     __fmul_rn(2.0f, __fsub_rn(x.z, y.z)), __fmul_rn(2.0f, __fsub_rn(x.w, y.w)));
}

// Stage ring shared by the producer and the consumers: stage s (a running
// count) lives in buffer s % kStages and completes phase (s / kStages) & 1.
template <int kSt, int kStageBytes>
struct RingT {
  uint32_t sbase, full0, empty0;
  __device__ __forceinline__ static int buf(int s) { return (unsigned)s % kSt; }
  __device__ __forceinline__ static uint32_t phase(int s) { return ((unsigned)s / kSt) & 1u; }
  __device__ __forceinline__ uint32_t stage(int s) const { return sbase + (uint32_t)(buf(s) * kStageBytes); }
  __device__ __forceinline__ void wait_full(int s) const {
    mbar_wait(full0 + 8u * buf(s), phase(s));
  }
  // Every consumer THREAD arrives (the empty barrier counts 32 per warp): each
  // thread's own release orders its reads of the stage before the producer's
  // refill.  (Lane 0 arriving after __syncwarp is equally correct under the
  // PTX memory model, and costs the same one warp instruction, but
  // compute-sanitizer racecheck reports it as WAR hazards on the stage
  // descriptor -- tools/repro/racecheck_mbarrier.cu.)
  __device__ __forceinline__ void release(int s, int lane) const {
    (void)lane;
    mbar_arrive(empty0 + 8u * buf(s));
  }
};

}  // namespace
}  // namespace sharp
