// TMEM-resident sm_100a kernel (SHARP_PATH_RES).  ONE
// persistent launch per batch, frames of up to ~10 Mpx.
//
// The two passes of the method -- pass 1: Sobel pEdge (L158-L172) summed for
// the global mean (L174); pass 2: everything else (downscale L130, upscale
// L140-L146, pError L148, 3x3 max/min L182, strength L178, overshoot
// L180-L212) -- both need pEdge.  The step kernel (kernels_tma.cu) computes
// the Sobel twice.  Here pass 1 leaves each tile's pEdge in TENSOR MEMORY
// (tcgen05.st: 8 pixels = 4 f16x2 words per lane and row; 256 KB per SM that
// no other part of this path uses) and pass 2 of the same tile, on the same
// warps, reads it back (tcgen05.ld) after the frame's mean is known: no second
// Sobel, no pEdge traffic to L2 or HBM.  The frame's input is re-read by pass
// 2 from L2 (the re-read follows its pass 1 closely): ~2 B/px of DRAM.
//
// ONE CTA per SM (all 512 TMEM columns) = three independent pipelines (each:
// 4 compute warps + a producer warp, its own smem stages and LUT buffers)
// + one table warp.  Tile = 960 columns (4 warp tiles of 240) x kT = 12 rows.
// Per pipeline the consumers process, in order,
//     P1(t0) P1(t1) P1(t2) P2(t0) P1(t3) P2(t1) P1(t4) P2(t2) ...
// (three TMEM slots of 48 columns per warp, tile k in slot k % 3), so between
// a tile's pass 1 and its pass 2 the pipeline does one full tile of other
// work while the rest of the GPU completes the frame's pass 1 and its table.
//
// Schedule: static -- pipeline v (of 3 x gridDim) takes positions v, v + 3
// gridDim, ... of the frame-major tile order.  A producer issues P1 of
// position k+2 before it waits for the table of position k, and a frame of
// <= 2 x (3 gridDim) tiles spans at most three positions of a pipeline, so by
// induction every awaited table completes (no deadlock; larger frames take
// the step kernel).
//
// Dependencies (the global barrier of L174): every pass-1 warp adds
// (1 << 40) + its partial sum to the frame's acc word.  The table warp of
// every SM walks the frames in order and, once a frame's acc shows all
// arrivals, builds 16-entry chunks of its table (lanes 0-15 A (p/m)^gamma,
// lanes 16-31 clamp(G exp(-p/(K m)), 0, 1), f64 rounded once: R9, R11); a
// producer needing a frame's table helps build the remaining chunks, then
// acquires it (an acquire load on its lane 0 or 1) and bulk-copies it into
// its LUT buffer as part of the pass-2 stage.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>

#include "device_common.cuh"
#include "kernels.h"
#include "tma_common.cuh"

namespace sharp {
namespace {
using namespace dev;

constexpr int kT = kTH;                 // rows per tile (pass 1 and pass 2)
// Pass 1 unpacks bytes as f16 subnormals (derive_w<.., true>; measured +1.8%
// on 1024 x 1080p): pEdge is kept in TMEM as pEdge * 2^-24, and the table key
// is 2^-3 + pEdge * 2^-24.
constexpr bool kDenorm = true;
constexpr float kLutKey = kDenorm ? 0.125f : 2097152.0f;
constexpr uint32_t kLutKeyBits = kDenorm ? 0x3E000000u : 0x4A000000u;
constexpr int kPipes = 3;               // independent pipelines per CTA (each: 4 compute warps + a producer)
constexpr int kCompute = kWarpsT * kPipes;       // 12 compute warps
constexpr int kThreadsR = 32 * (kCompute + kPipes + 1);  // + 3 producers + 1 table warp: ONE CTA per SM
constexpr int kRowsStage = kT + 8;               // stage rows: image rows R0-4 .. R0+15
constexpr int kRowsP1 = kT + 2;                  // pass-1 boxes: rows R0-1 .. R0+12 (at stage row 3)
constexpr int kSlotR = kPitch * kRowsStage;      // region A of one warp column
constexpr int kRegBR = kWarpsT * kSlotR;         // region B (the last warp column's right halo)
#ifndef SHARP_RES_STAGES
#define SHARP_RES_STAGES 3
#endif
constexpr int kResStages = SHARP_RES_STAGES;     // smem ring depth per pipeline
constexpr int kResStage = (kRegBR + kPitchB * kRowsStage + 127) / 128 * 128;
constexpr int kLutBufs = 2;
constexpr int kPipeLutOff = kResStages * kResStage;          // per pipeline: stages, LUT buffers, 16-B dummy
constexpr int kPipeDummy = kPipeLutOff + kLutBufs * kLutBytes;
constexpr int kPipeBytes = (kPipeDummy + 16 + 127) / 128 * 128;
constexpr int kResBarOff = kPipes * kPipeBytes;               // then full + empty barriers of every pipeline
constexpr int kResSmem = kResBarOff + kPipes * 16 * kResStages;
// TMEM: all 512 columns (one CTA per SM); compute warp w (pipeline w / 4)
// uses lane quarter w % 4 (the hardware's mapping) and columns 160 (w / 4)
// ..: three slots of 48 columns, slot q of a tile at +48 q, pEdge row j of
// the tile at +4 j.
constexpr uint32_t kTmemCols = 512;
constexpr int kWarpCols = 160;
constexpr int kSlots = 3;
constexpr int kSlotCols = 4 * kT;
static_assert(kSlots * kSlotCols <= kWarpCols && kPipes * kWarpCols <= (int)kTmemCols, "TMEM slots");
constexpr int kChunk = 16;                  // table entries per chunk: lanes 0-15 adj, 16-31 osc
constexpr int kChunks = kLut2 / kChunk;     // 48
constexpr int kAccShift = 40;
static_assert(kResStage % 128 == 0 && kPipeLutOff % 128 == 0 && (3 * kPitch) % 128 == 0, "TMA smem destinations");
static_assert(kResSmem <= 227 * 1024, "one CTA per SM");

using RRing = RingT<kResStages, kResStage>;

// Lane words of a warp column in this kernel's stage layout (cf. lane_row of
// tma_common.cuh: 44-row regions).  rb_shift: row offset of region B (the
// pass-1 region-B box lands at row 0 of region B but holds image row R0-1,
// stage row 3, so its base is moved 3 rows back).
__device__ __forceinline__ LaneRow lane_row_r(uint32_t stage, int wc, int lane, int rb_shift) {
  if (lane == 30) {
    if (wc == kWarpsT - 1) return LaneRow{stage + (uint32_t)(kRegBR - rb_shift * kPitchB), (uint32_t)kPitchB};
    return LaneRow{stage + (uint32_t)((wc + 1) * kSlotR + kCol0), (uint32_t)kPitch};
  }
  return LaneRow{stage + (uint32_t)(wc * kSlotR + kCol0 + 8 * (lane < 31 ? lane : -1)), (uint32_t)kPitch};
}
// The boxes of a CTA tile of nw warp columns into stage st: region A per
// column at row a_row, region B (when all 4 columns exist) at row 0.
__device__ __forceinline__ void tma_tiles_r(uint32_t st, const CUtensorMap *mapA, const CUtensorMap *mapB, int C0,
                                            int nw, int a_row, int r, int f, uint32_t bar, uint64_t policy) {
  for (int w = 0; w < nw; ++w)
    tma_box(st + w * kSlotR + a_row * kPitch, mapA, C0 + w * kTW - kCol0, r, f, bar, policy);
  if (nw == kWarpsT) tma_box(st + kRegBR, mapB, C0 + kWarpsT * kTW, r, f, bar, policy);
}
__device__ __forceinline__ uint32_t tile_bytes_r(int nw, int rows) {
  return (uint32_t)((nw * kPitch + (nw == kWarpsT ? kPitchB : 0)) * rows);
}
#ifndef SHARP_RES_CWAIT_NS
#define SHARP_RES_CWAIT_NS 0  // consumer stage waits: 0 = try_wait, else test_wait + back-off up to this (ns)
#endif
#ifndef SHARP_RES_HELP_NS
#define SHARP_RES_HELP_NS 256  // producer: sleep between looks while a table cannot be helped yet
#endif

#ifdef SHARP_DIAG_RES  // diagnostics build only: wait-cycle counters
__device__ unsigned long long g_rd[16];
__shared__ long long rd_tma[4], rd_lut[4];  // producer clocks per stage
#define RD_ADD(i, v) atomicAdd(&g_rd[i], (unsigned long long)(v))
#else
#define RD_ADD(i, v)
#endif

enum { kRP1 = 1, kRP2 = 3, kREnd = -1 };

struct ResParams {
  int W, H, n;
  int tiles_x, per_frame;  // CTA tiles per tile row / per frame
  int ntasks;              // n * per_frame
  // Static schedule: CTA c takes positions c, c + grid, c + 2 grid, ... of
  // the frame-major tile order; pad = 0: position == tile (per_frame <=
  // grid), else each frame occupies pad (= 2 grid) positions, its tiles
  // first (grid < per_frame <= 2 grid).  A frame thus spans at most two
  // positions of any CTA (the no-deadlock condition, header comment).
  int pad, npos;
  int rmax1;               // last row whose pEdge is summed (H - 2)
  Params prm;
  unsigned long long *acc;   // per frame: (pass-1 warp arrivals << 40) + sum of pEdge; zero on entry
  unsigned long long *sums;  // per frame: S
  double *means;             // per frame: S / (W H) (or the R8 alternative)
  float2 *luts;              // per frame: kLutSize entries {adj, osc}
  unsigned int *lut_next;    // per frame: chunks grabbed; zero on entry
  unsigned int *lut_done;    // per frame: chunks finished; zero on entry
  unsigned int *task_counter;
  uint8_t *out;
  size_t out_pitch, out_fs;
};

__device__ __forceinline__ bool mbar_test(uint32_t bar, uint32_t parity) {  // non-blocking
  uint32_t ok;
  asm volatile(
      "{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return __shfl_sync(0xffffffffu, ok, 0) != 0;
}

// ------------------------------------------------------------------- TMEM
__device__ __forceinline__ void tmem_st4(uint32_t taddr, const uint32_t v[4]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};" ::"r"(taddr), "r"(v[0]), "r"(v[1]),
               "r"(v[2]), "r"(v[3])
               : "memory");
}
__device__ __forceinline__ void tmem_ld4(uint32_t taddr, uint32_t v[4]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
               : "r"(taddr)
               : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// --------------------------------------------------------- pass 1 (warp)
// pEdge of rows R0 .. R0+kT-1 (smem row of image row r: r - R0 + 1) into
// TMEM row j = r - R0 of the slot, and the warp's partial sum of the Sobel
// body (rows 1..rmax1, columns 1..W-2; L160: the frame is 0).
// (aw: the warp column's lane words; sb: stage row of image row R0 - 1.)
// The sums: with the bytes unpacked as f16 subnormals, the f16 bit pattern of
// every pEdge value (<= 1530 < 2048 units of 2^-24) is the integer pEdge, so
// each f16x2 word is a u16x2 pair of pEdge values and the row sums are plain
// 32-bit integer adds, two pixels per add (halves stay < 2^16).
static_assert(kDenorm, "p1_tile sums the subnormal bit patterns");
__device__ __forceinline__ uint32_t p1_tile(const LaneRow &aw0, int sb, int W, int rmax1, int C0w, int R0, int lane,
                                            uint32_t tslot) {
  const int c0 = C0w + 8 * lane;
  const LaneRow aw{aw0.base + (uint32_t)sb * aw0.pitch, aw0.pitch};  // row offsets below are compile-time
  RowD ra = derive_w<false, kDenorm>(row_words(aw, 0), lane);
  RowD rb = derive_w<false, kDenorm>(row_words(aw, 1), lane);
  uint32_t acc[4] = {0u, 0u, 0u, 0u};  // per pair: (sum of the low pixel, of the high pixel)
#pragma unroll 1
  for (int m = 0; m < kT; m += 3) {
    uint32_t pe[3][4];
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      const RowD rc = derive_w<false, kDenorm>(row_words(aw, m + a + 2), lane);
      sobel(ra, rb, rc, pe[a]);
      tmem_st4(tslot + (uint32_t)(4 * (m + a)), pe[a]);
      ra = rb;
      rb = rc;
    }
    // rows 1 <= r <= rmax1 only (L160); warp-uniform (a vote)
    const int r = R0 + m;
    if (__all_sync(0xffffffffu, r >= 1 && r + 2 <= rmax1)) {
#pragma unroll
      for (int i = 0; i < 4; ++i) acc[i] = acc[i] + pe[0][i] + pe[1][i] + pe[2][i];
    } else {
#pragma unroll
      for (int a = 0; a < 3; ++a)
        if ((unsigned)(r + a - 1) < (unsigned)rmax1) {
#pragma unroll
          for (int i = 0; i < 4; ++i) acc[i] += pe[a][i];
        }
    }
  }
  // Sobel body columns only (L160: columns 0 and W-1 are frame); halo lanes
  // and lanes beyond the image add nothing.  Pair i holds x = 4 (i >> 1) +
  // (i & 1) (low half) and x + 2 (high half).
  uint32_t sum = 0;
  if (lane < 30) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int x = 4 * (i >> 1) + (i & 1);
      if (c0 + x >= 1 && c0 + x <= W - 2) sum += acc[i] & 0xffffu;
      if (c0 + x + 2 >= 1 && c0 + x + 2 <= W - 2) sum += acc[i] >> 16;
    }
  }
  tmem_wait_st();  // the slot's rows are in TMEM before this warp's pass 2 reads them
  return sum;
}

// --------------------------------------------------------- pass 2 (warp)
// Per image row: the centre values and the horizontal 3-max / 3-min (f16x2
// bit patterns; pass 2 needs no Sobel ingredients -- pEdge comes from TMEM).
struct RowM {
  uint32_t mx[4], mn[4], c[4];
};
__device__ __forceinline__ RowM derive_m(uint2 w, int lane) {
  const uint32_t E0 = hadd(prmt(w.x, kF16Bias, 0x4240), kMinus1024);  // (c0, c0+2)
  const uint32_t O0 = hadd(prmt(w.x, kF16Bias, 0x4341), kMinus1024);  // (c0+1, c0+3)
  const uint32_t E1 = hadd(prmt(w.y, kF16Bias, 0x4240), kMinus1024);  // (c0+4, c0+6)
  const uint32_t O1 = hadd(prmt(w.y, kF16Bias, 0x4341), kMinus1024);  // (c0+5, c0+7)
  const uint32_t PO = __shfl_sync(0xffffffffu, O1, (lane + 31) & 31);  // (c0-3, c0-1)
  const uint32_t NE = __shfl_sync(0xffffffffu, E0, (lane + 1) & 31);   // (c0+8, c0+10)
  const uint32_t p[4] = {E0, O0, E1, O1};
  const uint32_t l[4] = {prmt(PO, O0, 0x5432), E0, prmt(O0, O1, 0x5432), E1};
  const uint32_t r[4] = {O0, prmt(E0, E1, 0x5432), O1, prmt(E1, NE, 0x5432)};
  RowM d;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    d.c[i] = p[i];
    d.mx[i] = __vimax3_u16x2(l[i], p[i], r[i]);
    d.mn[i] = __vimin3_u16x2(l[i], p[i], r[i]);
  }
  return d;
}

// One output row (window rows a = r-1, b = r, c = r+1) from pEdge `pe_in`.
__device__ __forceinline__ void p2_row_res(const RowM &ra, const RowM &rb, const RowM &rc, const uint32_t pe_in[4],
                                           const float4 &V, const float4 &D0, const float4 &D1, uint32_t lut_q,
                                           uint8_t *orow, bool store, int r, int c0, int W, int H, bool edge_warp,
                                           int edge) {
  uint32_t pe[4] = {pe_in[0], pe_in[1], pe_in[2], pe_in[3]}, MX[4], MN[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    MX[i] = __vimax3_u16x2(ra.mx[i], rb.mx[i], rc.mx[i]);
    MN[i] = __vimin3_u16x2(ra.mn[i], rb.mn[i], rc.mn[i]);
  }
  // Upscale body (L146, R3) on pixel pairs; NU = -U, exact.
  const float2 nu01 = lin2(V.x, V.y, cwt(0), cwt(1));
  const float2 nu23 = lin2(V.y, V.z, cwt(2), cwt(3));
  const float2 nu45 = lin2(V.y, V.z, cwt(0), cwt(1));
  const float2 nu67 = lin2(V.z, V.w, cwt(2), cwt(3));
  float NU[8] = {nu01.x, nu01.y, nu23.x, nu23.y, nu45.x, nu45.y, nu67.x, nu67.y};
  if (r < 2 || r >= H - 2) {  // warp-uniform: upscale border lines, Sobel / overshoot frame rows
    ring_rows(NU, pe, MX, MN, D0, D1, r, c0, W, H, edge);
  } else if (edge_warp) {     // warp-uniform; only the edge lane changes
    ring_cols(NU, pe, MX, MN, D0, D1, r, H, edge);
  }
  float P[8], T8[8], osc[8];
#pragma unroll
  for (int x = 0; x < 8; ++x) {
    const int p = pair_of(x);
    const bool hi = half_of(x);
    // f32 bits of 2^21 + pEdge = 0x4A000000 + 8 k (kDenorm: pEdge * 2^-24 from
    // TMEM, 2^-3 + pEdge * 2^-24 = 0x3E000000 + 8 k): the byte offset of entry
    // k = pEdge / 2 scaled by the exponent (one FHADD, LDS [R + UR]).
    const uint32_t q8 = __float_as_uint(add_f32_f16(hi ? hi16(pe[p]) : lo16(pe[p]), kLutKey));
    const float2 L = lds_f2(q8 + lut_q);                                         // {adj, osc}
    const float E = add_f32_f16(hi ? hi16(rb.c[p]) : lo16(rb.c[p]), NU[x]);      // O - U (L148)
    P[x] = __fmaf_rn(L.x, E, -NU[x]);                                            // L178
    const float mxf = add_f32_f16(hi ? hi16(MX[p]) : lo16(MX[p]), 0.0f);
    const float mnf = add_f32_f16(hi ? hi16(MN[p]) : lo16(MN[p]), 0.0f);
    T8[x] = fminf(fmaxf(P[x], mnf), mxf);  // Fig. 8 branch target (max / min / P)
    osc[x] = L.y;
  }
  float F[8];
#pragma unroll
  for (int x = 0; x < 8; x += 2) {
    const float2 d = sub2(make_float2(P[x], P[x + 1]), make_float2(T8[x], T8[x + 1]));
    F[x] = __fmaf_rn(osc[x], d.x, T8[x]);  // osc max / osc min / P (R20)
    F[x + 1] = __fmaf_rn(osc[x + 1], d.y, T8[x + 1]);
  }
  const uint2 o = make_uint2(pack4_rni_u8(F[0], F[1], F[2], F[3]), pack4_rni_u8(F[4], F[5], F[6], F[7]));
  if (store) *reinterpret_cast<uint2 *>(orow) = o;
}

// Pass 2 of one warp tile (rows R0 .. R0+kT-1; smem row of image row r:
// r - R0 + 4), pEdge row j from TMEM column tslot + 4 j.
// (aw: the warp column's lane words; sb: stage row of image row R0 - 4.)
__device__ __forceinline__ void p2_tile(const LaneRow &aw0, int sb, uint32_t lut_q, uint32_t tslot,
                                        uint8_t *__restrict__ out, uint32_t out_pitch, int W, int H, int C0w, int R0,
                                        int lane) {
  const LaneRow aw{aw0.base + (uint32_t)sb * aw0.pitch, aw0.pitch};
  const int c0 = C0w + 8 * lane;
  const bool active = lane < 30 && c0 < W;
  const int edge = !active ? 0 : (c0 == 0 ? 1 : (c0 == W - 8 ? 2 : 0));
  const bool edge_warp = (C0w == 0) || (C0w <= W - 8 && W - 8 < C0w + kTW);
  // Vertical interpolation (L146, R3): V(r+1) = V(r) + 2 (D_{i+1} - D_i) on
  // r = 4i+2 .. 4i+5, restarted at r = 4i+2 (exact integers, x 128).
  const float4 Dp = dblock(aw, 0, lane);  // D row R0/4 - 1
  float4 D1 = dblock(aw, 4, lane);        // D row R0/4
  float4 D0 = Dp;
  float4 V = f4fma(5.0f, D1, f4fma(3.0f, Dp, make_float4(0.f, 0.f, 0.f, 0.f)));
  float4 slope = f4twice_diff(D1, Dp);
  RowM ra = derive_m(row_words(aw, 3), lane);
  RowM rb = derive_m(row_words(aw, 4), lane);
  uint8_t *orow = out + c0;
  const int rend = min(R0 + kT, H);
  const int rend_l = active ? rend : R0;
  // pEdge rows: the TMEM load of row j + 1 is issued while row j is computed
  uint32_t pe_next[4];
  tmem_ld4(tslot, pe_next);
#pragma unroll 1
  for (int r = R0; r < rend; r += 3) {
#pragma unroll
    for (int u = 0; u < 3; ++u) {
      const int rr = r + u;
      const int sm = rr - R0 + 4;
      uint32_t pe[4];
      tmem_wait_ld();
#pragma unroll
      for (int i = 0; i < 4; ++i) pe[i] = pe_next[i];
      tmem_ld4(tslot + (uint32_t)(4 * (rr - R0 + 1)), pe_next);  // (row kT: inside the warp's columns, unused)
      if ((rr & 3) == 0) {  // next D block row
        D0 = D1;
        D1 = dblock(aw, sm + 4, lane);
      } else if ((rr & 3) == 2) {  // next interpolation interval: D rows (k, k+1)
        V = f4fma(7.0f, D0, D1);
        slope = f4twice_diff(D1, D0);
      }
      const RowM rc = derive_m(row_words(aw, sm + 1), lane);
      p2_row_res(ra, rb, rc, pe, V, D0, D1, lut_q, orow, rr < rend_l, rr, c0, W, H, edge_warp, edge);
      V = f4add(V, slope);
      orow += out_pitch;
      ra = rb;
      rb = rc;
    }
  }
  tmem_wait_ld();  // the last prefetch lands before the slot is rewritten
}

// ------------------------------------------------- table build (producer)
// Chunk c of frame f's table: entries k = 32 c + lane (pEdge p = 2 k), f64
// rounded once (R9, R11), from the complete S.  All 32 lanes.
__device__ __forceinline__ void build_chunk(const ResParams &sp, int f, int c, unsigned long long S, int lane) {
  const int k = c * kChunk + (lane & (kChunk - 1)), p = 2 * k;
  const double mean = frame_mean(S, sp.W, sp.H, sp.prm.flags);  // L174 (R8)
  if (c == 0 && lane == 0) {
    sp.sums[f] = S;
    sp.means[f] = mean;
  }
  // the two transcendental evaluations of an entry on two lanes (half the
  // latency of a chunk: the table is on the frame's critical path)
  float *e = reinterpret_cast<float *>(sp.luts + (size_t)f * kLutSize + k);
  if (lane < kChunk) e[0] = p <= 1530 ? lut_adj(p, mean, sp.prm) : 0.0f;
  else e[1] = p <= 1530 ? lut_osc(p, mean, sp.prm) : 0.0f;
  __threadfence();
  __syncwarp();
  if (lane == 0) atomicAdd(&sp.lut_done[f], 1u);
  if (lane == 0) RD_ADD(5, 1);
}

// One step of work on frame f's table: returns 1 if it is complete, else
// builds one chunk if the frame's pass 1 is complete and a chunk is left
// (returns 0), else returns -1 (nothing to do now).  Warp-uniform.
__device__ __forceinline__ int table_step(const ResParams &sp, int f, int lane) {
  const unsigned long long arrivals = (unsigned long long)(sp.per_frame * kWarpsT) << kAccShift;
  unsigned done = 0;
  unsigned long long a = 0;
  if (lane == 0) {
    done = ld_relaxed_u32(&sp.lut_done[f]);
    if (done < (unsigned)kChunks) a = ld_relaxed_u64(&sp.acc[f]);
  }
  done = __shfl_sync(0xffffffffu, done, 0);
  if (done >= (unsigned)kChunks) return 1;
  a = __shfl_sync(0xffffffffu, a, 0);
  if ((a & ~((1ull << kAccShift) - 1)) != arrivals) return -1;
  int c = 0;
  if (lane == 0) c = ld_relaxed_u32(&sp.lut_next[f]) < (unsigned)kChunks ? (int)atomicAdd(&sp.lut_next[f], 1u) : kChunks;
  c = __shfl_sync(0xffffffffu, c, 0);
  if (c >= kChunks) return -1;
  build_chunk(sp, f, c, a & ((1ull << kAccShift) - 1), lane);
  return 0;
}

// Acquire frame f's complete table on lane `who` (an acquire LOAD, not a
// fence.acq_rel, which would also wait for the thread's in-flight TMA
// loads), then order the thread's later bulk copy (async proxy) after it.
__device__ __forceinline__ void acquire_table(const ResParams &sp, int f, int lane, int who) {
  if (lane == who) {
    while (ld_acquire(&sp.lut_done[f]) < (unsigned)kChunks) {
    }
    fence_proxy_async_global();
  }
  __syncwarp();
}

// Returns once frame f's table is complete; meanwhile builds chunks of it
// (once its pass 1 is complete).  Warp-uniform (all 32 producer lanes).
// A frame whose table never completes (a bug, or a broken no-deadlock
// condition) must not hang the device: the dependency waits trap after 10 s.
__device__ __forceinline__ void watchdog(unsigned long long t0) {
  if (gtime_ns() - t0 > 10000000000ull) __trap();
}

__device__ __forceinline__ void ensure_table(const ResParams &sp, int f, int lane) {
  const unsigned long long wd0 = gtime_ns();
#ifdef SHARP_DIAG_NO_TABLE_WAIT  // timing experiment only: wrong output
  return;
#endif
  const unsigned long long arrivals = (unsigned long long)(sp.per_frame * kWarpsT) << kAccShift;
#ifdef SHARP_DIAG_RES
  long long t_first_complete = 0, t_enter = clock64();
  int iters = 0;
#endif
  for (;;) {
#ifdef SHARP_DIAG_RES
    ++iters;
#endif
    unsigned done = 0;
    unsigned long long a = 0;
    if (lane == 0) {
      done = ld_relaxed_u32(&sp.lut_done[f]);
      if (done < (unsigned)kChunks) a = ld_relaxed_u64(&sp.acc[f]);
    }
    done = __shfl_sync(0xffffffffu, done, 0);
    if (done >= (unsigned)kChunks) break;
    a = __shfl_sync(0xffffffffu, a, 0);
    if ((a & ~((1ull << kAccShift) - 1)) == arrivals) {
#ifdef SHARP_DIAG_RES
      if (!t_first_complete) t_first_complete = clock64();
#endif
      int c = 0;
      if (lane == 0)
        c = ld_relaxed_u32(&sp.lut_next[f]) < (unsigned)kChunks ? (int)atomicAdd(&sp.lut_next[f], 1u) : kChunks;
      c = __shfl_sync(0xffffffffu, c, 0);
      if (c < kChunks) {
        build_chunk(sp, f, c, a & ((1ull << kAccShift) - 1), lane);
        continue;
      }
    }
    __nanosleep(SHARP_RES_HELP_NS);
    watchdog(wd0);
  }
#ifdef SHARP_DIAG_RES
  if (lane == 0) {
    const long long now = clock64();
    if (iters == 1) RD_ADD(8, 1);  // table complete at the first look
    if (t_first_complete) {
      RD_ADD(9, t_first_complete - t_enter);  // waiting for the frame's pass 1
      RD_ADD(10, now - t_first_complete);     // then for the table
      RD_ADD(11, 1);
    }
  }
#endif
  __syncwarp();
}

// ============================================================== the kernel
__global__ void __launch_bounds__(kThreadsR, 1)
    res_kernel(const __grid_constant__ CUtensorMap map1A, const __grid_constant__ CUtensorMap map1B,
               const __grid_constant__ CUtensorMap map2A, const __grid_constant__ CUtensorMap map2B, ResParams sp) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ int4 stage_task[kPipes][kResStages];  // {type, frame, C0, R0}
  __shared__ int2 stage_aux[kPipes][kResStages];   // {TMEM slot, LUT buffer}
  __shared__ uint32_t tmem_base;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t sbase = smem_u32(smem);
  // pipeline of this warp: compute warps 4p..4p+3, producer warp kCompute + p
  const int pipe = warp < kCompute ? warp / kWarpsT : (warp < kCompute + kPipes ? warp - kCompute : 0);
  const uint32_t pbase = sbase + (uint32_t)(pipe * kPipeBytes);
  const uint32_t bars = sbase + kResBarOff + (uint32_t)(pipe * 16 * kResStages);
  const RRing ring{pbase, bars, bars + 8 * kResStages};
  const uint32_t lutbase = pbase + kPipeLutOff;

  if (warp == 0) {  // TMEM for the pEdge slots (warp 0 allocates and frees)
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)),
                 "n"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < kPipes * kResStages; ++i) {
      const uint32_t b0 = sbase + kResBarOff + (uint32_t)((i / kResStages) * 16 * kResStages);
      mbar_init(b0 + 8 * (i % kResStages), 1);
      mbar_init(b0 + 8 * kResStages + 8 * (i % kResStages), 32 * kWarpsT);  // every consumer thread arrives
    }
    fence_barrier_init();
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");

  if (warp == kCompute + kPipes) {
    // --------------------------------------------------------- table warp
    // Builds chunks of every frame's table as soon as the frame's pass 1 is
    // complete (all SMs' table warps in parallel: a frame's 48 chunks take
    // about one f64 pow latency).  The tables are the dependency of every
    // pass-2 tile, so their build must not wait for the producers that need
    // them (measured: 5 us per frame when only the waiting producers built).
    for (int f = 0; f < sp.n; ++f) {
      const unsigned long long wd0 = gtime_ns();
      for (;;) {
        watchdog(wd0);
        const int st = table_step(sp, f, lane);
        if (st == 1) break;                                      // complete
        if (st < 0) {
          unsigned next = 0;
          if (lane == 0) next = ld_relaxed_u32(&sp.lut_next[f]);
          if (__shfl_sync(0xffffffffu, next, 0) >= (unsigned)kChunks) break;  // all chunks taken
          __nanosleep(SHARP_RES_HELP_NS);
        }
      }
    }
    return;
  }
  if (warp >= kCompute) {
    // ------------------------------------------------------------ producer
    // (one per pipeline: a "virtual CTA" v = kPipes * blockIdx.x + pipe of a
    // grid of kPipes * gridDim.x, with its own stages and LUT buffers)
    const uint64_t pol_keep = policy_evict_last(), pol_drop = policy_evict_first();
    int s = 0;                                        // stages filled
    // per LUT buffer b (scalars, not arrays: no local memory): the last stage
    // that used it and the frame whose table it holds
    int lut_last0 = -kResStages, lut_last1 = -kResStages, lut_frame0 = -1, lut_frame1 = -1;
    int lut_prev = 1;                                 // buffer of the previous pass-2 tile
    const int vgrid = kPipes * gridDim.x;
    int pos = kPipes * blockIdx.x + pipe;
    auto next_tile = [&]() -> int {  // this pipeline's next tile (static schedule), or ntasks
      while (pos < sp.npos) {
        const int p = pos;
        pos += vgrid;
        if (!sp.pad) return p;
        const int f = p / sp.pad, i = p - f * sp.pad;
        if (i < sp.per_frame) return f * sp.per_frame + i;
      }
      return sp.ntasks;
    };
    auto begin_stage = [&]() -> int {  // next stage's buffer, once its consumers released it
      const int b = RRing::buf(s);
#ifdef SHARP_DIAG_RES
      const long long w0 = clock64();
#endif
      if (s >= kResStages) mbar_wait(ring.empty0 + 8u * b, RRing::phase(s) ^ 1u);
#ifdef SHARP_DIAG_RES
      if (lane == 0) RD_ADD(6, clock64() - w0);
#endif
      return b;
    };
    auto tile_of = [&](int t, int &f, int &C0, int &R0, int &nw) {
      f = t / sp.per_frame;
      const int i = t - f * sp.per_frame, ty = i / sp.tiles_x;
      C0 = (i - ty * sp.tiles_x) * kCtaCols;
      R0 = ty * kT;
      nw = 0;
#pragma unroll
      for (int w = 0; w < kWarpsT; ++w) nw += (C0 + w * kTW < sp.W);
    };
    auto issue_p1 = [&](int t, int q) {
      int f, C0, R0, nw;
      tile_of(t, f, C0, R0, nw);
      const int b = begin_stage();
      if (lane == 0) {
        const uint32_t full = ring.full0 + 8u * b, st = ring.stage(s);
        stage_task[pipe][b] = make_int4(kRP1, f, C0, R0);
        stage_aux[pipe][b] = make_int2(q, 0);
        mbar_expect_tx(full, tile_bytes_r(nw, kRowsP1));
        tma_tiles_r(st, &map1A, &map1B, C0, nw, 3, R0 - 1, f, full, pol_keep);  // stage row 3 = image row R0-1
      }
      __syncwarp();
      ++s;
    };
    auto issue_p2 = [&](int t, int q) {
      int f, C0, R0, nw;
      tile_of(t, f, C0, R0, nw);
      // LUT buffer: the one already holding frame f's table, else the one the
      // previous pass-2 tile did not use (free once the stage that last read
      // it is released)
      const int lb = lut_frame0 == f ? 0 : lut_frame1 == f ? 1 : (lut_prev ^ 1);
      const bool copy = (lb ? lut_frame1 : lut_frame0) != f;
      // While the stage is still in use: help build frame f's table (its
      // builders are the producers that wait for it), and once it is complete
      // acquire it -- so that when the stage frees, the table copy and the
      // tile loads go out at once (each global round trip here costs ~0.5 us
      // under load; measured).
      bool ready = !copy;
#ifdef SHARP_DIAG_NO_TABLE_WAIT
      ready = true;
#endif
      if (s >= kResStages) {
        const uint32_t eb = ring.empty0 + 8u * RRing::buf(s), par = RRing::phase(s) ^ 1u;
        const unsigned long long wd0 = gtime_ns();
        while (!ready && !mbar_test(eb, par)) {
          watchdog(wd0);
          const int st = table_step(sp, f, lane);
          if (st == 1) {
            acquire_table(sp, f, lane, 0);
            ready = true;
          } else if (st < 0) {
            __nanosleep(SHARP_RES_HELP_NS);
          }
        }
      }
      const int b = begin_stage();
      const uint32_t full = ring.full0 + 8u * b, st = ring.stage(s);
      const uint32_t lut_dst = lutbase + (uint32_t)(lb * kLutBytes);
      const float2 *lut_src = sp.luts + (size_t)f * kLutSize;
      if (lane == 0) {
        stage_task[pipe][b] = make_int4(kRP2, f, C0, R0);
        stage_aux[pipe][b] = make_int2(q, lb);
        const int tl = lb ? lut_last1 : lut_last0;
        if (copy && tl > s - kResStages) mbar_wait(ring.empty0 + 8u * RRing::buf(tl), RRing::phase(tl));
        mbar_expect_tx(full, tile_bytes_r(nw, kRowsStage) + (copy ? (uint32_t)kLutBytes : 0u));
#ifdef SHARP_DIAG_RES
        rd_tma[b] = clock64();
        rd_lut[b] = rd_tma[b];
#endif
        if (copy && ready) bulk_copy(lut_dst, lut_src, kLutBytes, full);
        tma_tiles_r(st, &map2A, &map2B, C0, nw, 0, R0 - 4, f, full, pol_drop);  // (loads need no table)
      }
      if (copy && !ready) {
#ifdef SHARP_DIAG_RES
        const long long w0 = clock64();
#endif
        ensure_table(sp, f, lane);  // frame f's pass 1 complete, its table built (helping)
#ifdef SHARP_DIAG_RES
        if (lane == 0) RD_ADD(4, clock64() - w0);
#endif
        // lane 1: a fence would also wait for lane 0's in-flight tile loads
        acquire_table(sp, f, lane, 1);
        if (lane == 1) bulk_copy(lut_dst, lut_src, kLutBytes, full);
#ifdef SHARP_DIAG_RES
        if (lane == 1) rd_lut[b] = clock64();
#endif
      }
      if (copy) (lb ? lut_frame1 : lut_frame0) = f;
      __syncwarp();
      (lb ? lut_last1 : lut_last0) = s;
      lut_prev = lb;
      ++s;
    };
    // P1(t0) P1(t1) then [P2(t_k) P1(t_{k+2})]...: a tile is grabbed only
    // after the table of the CTA's oldest unfinished tile is complete.
    int t0 = next_tile();
    if (t0 < sp.ntasks) issue_p1(t0, 0);
    int t1 = t0 < sp.ntasks ? next_tile() : sp.ntasks;
    if (t1 < sp.ntasks) issue_p1(t1, 1);
    int t2 = t1 < sp.ntasks ? next_tile() : sp.ntasks;
    if (t2 < sp.ntasks) issue_p1(t2, 2);
    for (int q = 0; t0 < sp.ntasks; q = q + 1 == kSlots ? 0 : q + 1) {
      issue_p2(t0, q);
      const int tn = t2 < sp.ntasks ? next_tile() : sp.ntasks;
      if (tn < sp.ntasks) issue_p1(tn, q);
      t0 = t1;
      t1 = t2;
      t2 = tn;
    }
    // end stage: the descriptor is published through a (16-byte) bulk copy's
    // complete_tx like every data stage
    const int b = begin_stage();
    if (lane == 0) {
      const uint32_t full = ring.full0 + 8u * b;
      stage_task[pipe][b] = make_int4(kREnd, 0, 0, 0);
      mbar_expect_tx(full, 16u);
      bulk_copy(pbase + kPipeDummy, sp.luts, 16u, full);
    }
    return;
  }

  // -------------------------------------------------------------- consumers
  // warp wc (240 columns) of its pipeline's tiles; TMEM lane quarter wc,
  // columns 160 pipe + 48 slot ..
  const int wc = warp % kWarpsT;
  const uint32_t tmem_w = tmem_base + ((uint32_t)(32 * wc) << 16) + (uint32_t)(pipe * kWarpCols);
  const int W = sp.W, H = sp.H;
  for (int s = 0;; ++s) {
    const int b = RRing::buf(s);
#ifdef SHARP_DIAG_RES
    const long long w0 = clock64();
#endif
    ring.wait_full(s);
    const int4 d = stage_task[pipe][b];
    const int2 aux = stage_aux[pipe][b];
#ifdef SHARP_DIAG_RES
    if (lane == 0) {
      const long long now = clock64();
      RD_ADD(d.x == kRP1 ? 0 : 2, now - w0);
      RD_ADD(d.x == kRP1 ? 1 : 3, 1);
      if (d.x == kRP2 && warp == 0 && now - w0 > 1000) {  // a P2 wait: issue-to-ready of tiles / table copy
        RD_ADD(14, now - rd_tma[b]);
        RD_ADD(15, now - rd_lut[b]);
        RD_ADD(13, 1);
      }
    }
#endif
    if (d.x == kREnd) break;
    const int f = d.y, C0w = d.z + wc * kTW, R0w = d.w;
    const uint32_t tslot = tmem_w + (uint32_t)(aux.x * kSlotCols);
    if (d.x == kRP1) {
      const uint32_t acc =
          C0w < W ? p1_tile(lane_row_r(ring.stage(s), wc, lane, 3), 3, W, sp.rmax1, C0w, R0w, lane, tslot) : 0u;
      // Reduction (sec. V-C): warp REDUX, one u64 atomic per warp adding the
      // arrival and the partial in one word (the table builders wait on it).
      const uint32_t ws = __reduce_add_sync(0xffffffffu, acc);
      if (lane == 0) atomicAdd(&sp.acc[f], (1ull << kAccShift) + (unsigned long long)ws);
    } else if (C0w < W && R0w < H) {
      // LDS address of entry k = pEdge/2: f32 bits of (2^21 + pEdge) + lut_q
      // (warp-uniform by the vote: folded into LDS [R + UR]).
      const uint32_t lut_q =
          lutbase + (__any_sync(0xffffffffu, aux.y) ? (uint32_t)kLutBytes : 0u) - kLutKeyBits;
      p2_tile(lane_row_r(ring.stage(s), wc, lane, 0), 0, lut_q, tslot,
              sp.out + (size_t)f * sp.out_fs + (size_t)R0w * sp.out_pitch, (uint32_t)sp.out_pitch, W, H, C0w, R0w,
              lane);
    }
    ring.release(s, lane);
  }
  // teardown: every consumer warp's TMEM accesses are complete
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  asm volatile("bar.sync 1, %0;" ::"n"(kCompute * 32) : "memory");
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(kTmemCols));
  }
}

// ----------------------------------------------------------------- host side
constexpr int kMaxDevices = 64;
std::atomic<int> g_res_grid[kMaxDevices];  // resident CTAs x SMs per device (preload_res)
int cur_dev() {
  int dev = 0;
  cudaGetDevice(&dev);
  return (dev >= 0 && dev < kMaxDevices) ? dev : 0;
}

}  // namespace

int res_grid() { return g_res_grid[cur_dev()].load(std::memory_order_relaxed); }

bool res_supported(int W, int H, int n) {
  (void)n;
  const long long per_frame = (long long)((W + kCtaCols - 1) / kCtaCols) * ((H + kT - 1) / kT);
  const int grid = res_grid();
  return grid > 0 && per_frame <= 2ll * kPipes * grid;
}

cudaError_t launch_batch_res(const BatchLaunch &a, int W, int H, const Params &p, cudaStream_t stream) {
  if (a.n <= 0) return cudaSuccess;
  if (!res_supported(W, H, a.n) || !a.lut_next) return cudaErrorNotSupported;
  const size_t ip = a.in_pitch ? a.in_pitch : (size_t)W, ifs = a.in_fs ? a.in_fs : ip * H;
  CUtensorMap m1A, m1B, m2A, m2B;
  if (!make_map(&m1A, a.in, a.n, W, H, ip, ifs, kPitch, kRowsP1) ||
      !make_map(&m1B, a.in, a.n, W, H, ip, ifs, kPitchB, kRowsP1) ||
      !make_map(&m2A, a.in, a.n, W, H, ip, ifs, kPitch, kRowsStage) ||
      !make_map(&m2B, a.in, a.n, W, H, ip, ifs, kPitchB, kRowsStage))
    return cudaErrorInvalidValue;
  ResParams sp;
  sp.W = W;
  sp.H = H;
  sp.n = a.n;
  sp.tiles_x = (W + kCtaCols - 1) / kCtaCols;
  sp.per_frame = sp.tiles_x * ((H + kT - 1) / kT);
  sp.ntasks = a.n * sp.per_frame;
  sp.rmax1 = H - 2;
  sp.prm = p;
  sp.acc = a.acc;
  sp.sums = a.sums;
  sp.means = a.means;
  sp.luts = a.luts;
  sp.lut_next = a.lut_next;
  sp.lut_done = a.lut_done;
  sp.task_counter = a.task_counter;
  sp.out = a.out;
  sp.out_pitch = a.out_pitch ? a.out_pitch : (size_t)W;
  sp.out_fs = a.out_fs ? a.out_fs : sp.out_pitch * (size_t)H;
  int grid = std::min(res_grid(), (sp.ntasks + kPipes - 1) / kPipes);
  if (a.grid_cap > 0) grid = std::min(grid, a.grid_cap);
  if (sp.per_frame > 2 * kPipes * grid) return cudaErrorNotSupported;  // the no-deadlock bound (header comment)
  // (dense order: with three pEdge slots a frame may span three positions of
  // a CTA -- P2 of position k follows P1 of position k+2 -- so up to 2 x grid
  // tiles need no padding)
  sp.pad = 0;
  sp.npos = sp.pad ? a.n * sp.pad : sp.ntasks;
  // A COOPERATIVE launch: the static schedule needs every CTA resident at
  // once (a CTA waits for tables that other CTAs' pass-1 tiles complete), and
  // a cooperative launch is scheduled only as a whole -- two of these kernels
  // on concurrent streams, or beside a persistent step kernel, cannot each
  // hold part of the SMs and wait on their missing halves.
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreadsR);
  cfg.dynamicSmemBytes = kResSmem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, res_kernel, m1A, m1B, m2A, m2B, sp);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

#ifdef SHARP_DIAG_RES
extern "C" int sharp_debug_res_grid() { return res_grid(); }
extern "C" int sharp_debug_res_occ(int *out) {
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, res_kernel);
  out[0] = fa.numRegs;
  out[1] = (int)fa.sharedSizeBytes;
  out[2] = fa.maxDynamicSharedSizeBytes;
  out[3] = kResSmem;
  int r = -1;
  out[4] = (int)cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, res_kernel, kThreadsR, kResSmem);
  out[5] = r;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, res_kernel, kThreadsR, 0);
  out[6] = r;
  out[7] = fa.maxThreadsPerBlock;
  return 0;
}
extern "C" int sharp_debug_res(unsigned long long *out, int reset) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, g_rd, sizeof(g_rd));
  if (reset) {
    static const unsigned long long z[16] = {};
    cudaMemcpyToSymbol(g_rd, z, sizeof(z));
  }
  return 0;
}
#endif

cudaError_t preload_res() {
  cudaError_t e;
  if ((e = cudaFuncSetAttribute(res_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kResSmem)) != cudaSuccess)
    return e;
  const int dev = cur_dev();
  // Resident CTAs per SM.  (cudaOccupancyMaxActiveBlocksPerMultiprocessor
  // reports 1 for any kernel using tcgen05.alloc, while 3 CTAs of 160 threads
  // with 128 TMEM columns each do run concurrently on an SM -- measured; so
  // the limit is computed from the register file, shared memory, threads and
  // TMEM columns.  It must not overestimate: the CTAs wait on each other.)
  cudaDeviceProp pr;
  cudaFuncAttributes fa;
  if ((e = cudaGetDeviceProperties(&pr, dev)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&fa, res_kernel)) != cudaSuccess) return e;
  const int warps = kThreadsR / 32;
  const int regs_warp = ((fa.numRegs * 32 + 255) / 256) * 256;
  const int by_regs = pr.regsPerMultiprocessor / (regs_warp * warps);
  const int by_smem =
      (int)(pr.sharedMemPerMultiprocessor / (kResSmem + fa.sharedSizeBytes + pr.reservedSharedMemPerBlock));
  const int by_threads = pr.maxThreadsPerMultiProcessor / kThreadsR;
  int res = std::min(std::min(by_regs, by_smem), std::min(by_threads, pr.maxBlocksPerMultiProcessor));
  res = std::min(res, (int)(512 / kTmemCols));
  res = std::min(res, 1);  // one CTA per SM (it allocates all 512 TMEM columns)
  const int sms = pr.multiProcessorCount;
  g_res_grid[dev].store(std::max(1, res) * (sms > 0 ? sms : 148));
  return cudaSuccess;
}

}  // namespace sharp
