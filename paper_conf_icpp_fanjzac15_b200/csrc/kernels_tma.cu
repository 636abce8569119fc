// TMA-staged, warp-specialised, dynamically scheduled sm_100a "step" kernel
// (the main path; needs W % 16 == 0 and 16-byte aligned frames -- the TMA
// tensor-map rules).  ONE launch processes a whole batch of frames.
//
// Persistent CTAs (3 per SM) grab tasks from a global counter.  The task list
// is a sequence of rounds; round rho holds
//   [pass-1 tasks of frame rho][LUT tasks of frame rho-L1][pass-2 tasks of frame rho-L2]
//   * pass 1: Sobel (L158-L172) + reduction (L174, sec. V-C): warp-shuffle
//     reduction and one packed u64 atomic per warp (arrival count | partial S);
//   * LUT: per-frame tables adj(p) = A (p/m)^gamma (strength, L178) and
//     osc(p) = clamp(G exp(-p/(K m)), 0, 1) (oscStrength, L184), 128 entries
//     per task, f64 rounded once (R9, R11), once the frame's S is complete;
//   * pass 2: the fused per-pixel pipeline (downscale L130, upscale L140-L146,
//     pError L148, Sobel, 3x3 max/min L182, strength lookup, preliminary
//     L178, overshoot L180-L212) -> u8, once the frame's LUT is written.
// The lags L1 < L2 make the dependencies (checked by the producer before it
// fills a stage) normally complete long before they are needed; a frame's
// input is re-read by pass 2 from L2 (pass-1 loads carry evict_last).
//
// CTA = 4 compute warps + 1 producer warp.  A pass-1/2 task is a column of
// CTA tiles ("sub-tiles", one smem stage each: 4 warp tiles side by side of
// 240 output columns x 12 rows for pass 2, x 18 rows for pass 1): 4 pass-2 /
// 2 pass-1 sub-tiles per task in big launches, the warps carrying their row
// window and sums from one sub-tile to the next.  The producer grabs its next
// task while issuing the current task's last stage, so the dependency lags
// stay short and a frame is still in L2 when its pass 2 re-reads it.  The producer issues one 256-column TMA box
// per warp tile (out-of-image pixels are zero-filled: no bounds checks in the
// pixel loops) plus a bulk copy of the frame's LUT, into one of two smem stages
// guarded by full/empty mbarriers -- no CTA-wide barrier in the steady state.
// Each lane owns 8 adjacent columns and walks down the rows with a 3-row
// window unrolled by 3 (no register moves); lanes 30 and 31 fetch the
// right/left halo columns and hand them out by shuffle.  The 2-pixel image
// ring (upscale border lines L140-L142, Sobel frame L160, overshoot frame
// L208) is handled in the same vectorised loop: a warp-uniform branch for
// the ring rows, lane-predicated overrides for the ring columns.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <atomic>

#include "device_common.cuh"
#include "kernels.h"
#include "tma_common.cuh"

namespace sharp {
namespace {
using namespace dev;

constexpr int kCtasPerSm = 3;  // smem ~67 KB per CTA
#ifndef SHARP_LB_CTAS
#define SHARP_LB_CTAS kCtasPerSm
#endif
constexpr int kLutPerTask = 32 * kWarpsT;      // LUT entries per LUT task (one per thread)
constexpr int kLutTasks = kLut2 / kLutPerTask;
constexpr int kTH1 = 18;              // pass-1 output rows per warp tile (fits the same slot)
constexpr int kRows1 = kTH1 + 2;      // pass-1 box rows: R0-1 .. R0+kTH1
// A pass-1 task is kSub1 vertically adjacent sub-tiles (one stage each); the
// warps carry their row window and sums from one to the next (no re-derived
// warm-up rows, one reduction per task).  Sums stay < 2^16 per u16 half:
// kSub1 * kTH1 * 1530 < 65536.
#ifndef SHARP_P1_SUB
#define SHARP_P1_SUB 2
#endif
constexpr int kSub1 = SHARP_P1_SUB;
static_assert(kSub1 * kTH1 * 1530 < 65536, "pass-1 u16 sums");
static_assert(kRows1 <= kRows2 && kSlot % 128 == 0, "pass-1 tiles fit the slots");
// A pass-2 task is kSub vertically adjacent CTA tiles ("sub-tiles") of one
// frame: each sub-tile fills one stage, the frame's LUT is copied once per
// task into one of two LUT buffers (task parity), and the warps carry their
// row window, D rows and interpolation state from one sub-tile to the next.
#ifndef SHARP_P2_SUB
#define SHARP_P2_SUB 4
#endif
constexpr int kSub = SHARP_P2_SUB;
// Launches of fewer frames take the compact task order (no lag rounds).
#ifndef SHARP_COMPACT_N
#define SHARP_COMPACT_N 32
#endif
constexpr int kCompactN = SHARP_COMPACT_N;
#ifndef SHARP_STAGES
#define SHARP_STAGES 2  // measured: 3 stages +0.3%, 2 stages (this layout) +0.6% vs the old layout
#endif
constexpr int kStages = SHARP_STAGES;          // smem ring depth
// Uniform-pitch stage layout: slot w holds one 256-column box; warps 0..2
// load columns C0w-16 .. C0w+239 (own columns at slot column kCol0), the last
// warp loads C0w .. C0w+255 (own columns at slot column 0, its right halo
// C0w+240.. in its own slot), so every lane -- halo lanes included -- reads
// its rows at pitch kPitch: row addresses are one base register plus
// immediates, and no 16-column region-B box is needed.
constexpr int kStage = kWarpsT * kSlot;  // one stage
__device__ __forceinline__ int own_col(int w) { return w == kWarpsT - 1 ? 0 : kCol0; }
struct LaneRowC {
  uint32_t base;
};
__device__ __forceinline__ LaneRowC lane_row_s(uint32_t stage, int warp, int lane) {
  const uint32_t own = stage + (uint32_t)(warp * kSlot + own_col(warp));
  if (lane < 30) return LaneRowC{own + 8u * (uint32_t)lane};
  if (lane == 30)  // right halo C0w+240..247
    return LaneRowC{warp == kWarpsT - 1 ? own + (uint32_t)kTW
                                        : stage + (uint32_t)((warp + 1) * kSlot + own_col(warp + 1))};
  // lane 31: left halo C0w-8..C0w-1 (the previous warp's slot for the last warp)
  return LaneRowC{warp == kWarpsT - 1 ? stage + (uint32_t)((warp - 1) * kSlot + kCol0 + kTW - 8) : own - 8u};
}
__device__ __forceinline__ uint2 row_words(const LaneRowC &a, int s) { return lds_u64(a.base + (uint32_t)(s * kPitch)); }
__device__ __forceinline__ float4 dblock(const LaneRowC &a, int s, int lane) {
  const uint32_t o = a.base + (uint32_t)(s * kPitch);
  const uint2 r0 = lds_u64(o), r1 = lds_u64(o + kPitch), r2 = lds_u64(o + 2 * kPitch), r3 = lds_u64(o + 3 * kPitch);
  const float d0 = (float)blk4(r0.x, r1.x, r2.x, r3.x);
  const float d1 = (float)blk4(r0.y, r1.y, r2.y, r3.y);
  const float dm1 = __shfl_sync(0xffffffffu, d1, (lane + 31) & 31);
  const float d2 = __shfl_sync(0xffffffffu, d0, (lane + 1) & 31);
  return make_float4(dm1, d0, d1, d2);
}
__device__ __forceinline__ uint32_t tile_bytes_s(int nw, int rows) { return (uint32_t)(nw * kPitch * rows); }
__device__ __forceinline__ void tma_tiles_s(uint32_t st, const CUtensorMap *mapA, const CUtensorMap *, int C0, int nw,
                                            int r, int f, uint32_t bar, uint64_t policy) {
  for (int w = 0; w < nw; ++w) tma_box(st + w * kSlot, mapA, C0 + w * kTW - own_col(w), r, f, bar, policy);
}
using LR = LaneRowC;
constexpr int kLutOff = kStages * kStage;      // two LUT buffers after the stages
constexpr int kBarOff = kLutOff + 2 * kLutBytes;
constexpr int kSmem = kBarOff + 16 * kStages;  // full + empty barrier per stage
static_assert(kSlot % 128 == 0 && kStage % 128 == 0, "TMA smem destinations must be 128-B aligned");
static_assert(kTH % 3 == 0 && kTH % 4 == 0, "row loop is unrolled by 3, D blocks are 4 rows");
static_assert(kTH1 % 3 == 0, "pass-1 tiles (3-row loop)");
static_assert(kLut2 % kLutPerTask == 0 && kLut2 <= kLutSize && 2 * (kLut2 - 1) >= 1530, "LUT tasks");

// ------------------------------------------------------------------ tasks
struct Geo {
  int W, H;        // the whole image (ring rows, Sobel frame, mean denominator)
  int tiles_x;     // CTA tiles per row band (ceil(W / 960))
  int per_frame;   // pass-2 tasks per frame (sub sub-tiles of kTH rows each)
  int sub;         // sub-tiles per pass-2 task (kSub; 1 when a launch has too few tasks to fill the GPU)
  int per_frame1;  // pass-1 CTA tiles per frame (th1 rows)
  int th1;         // pass-1 rows per sub-tile: kTH1, or 9 when a launch has too few tiles
  int sub1;        // pass-1 sub-tiles per task (kSub1, or 1 with short sub-tiles)
  // Rows processed: [row_lo, row_hi) of the image (the whole image, or one
  // row band, sec. 8(e)); the tensor map's row 0 is image row y0 (a band's
  // buffer starts with its upper halo); rmax1 = min(H-2, row_hi-1) is the
  // last row whose pEdge this launch sums.
  int row_lo, row_hi, y0, rmax1;
};

// The task sequence is a list of rounds; round rho holds
//   [pass-1 tasks of frame rho][LUT tasks of frame rho-L1][pass-2 tasks of frame rho-L2]
// (slots for frames outside [0, n) are empty tasks).  The lags L1 < L2 are
// chosen so that a frame's dependencies were grabbed long before (they are
// normally complete when the producer checks them).
enum TaskType { kEmpty = 0, kP1 = 1, kLut = 2, kP2 = 3, kHalo = 4, kEnd = -1 };
struct StepParams {
  Geo g;
  int mode;       // kStepAll, or a row band's kStepPass1 / kStepPass2
  int compact;    // kStepAll with < 4 frames: [all pass 1][all LUT][all pass 2], no lag rounds
  int n;          // frames
  int L1, L2;     // round lags of the LUT and pass-2 tasks
  int per_round;  // 2 * per_frame + kLutTasks
  int ntasks;     // (n + L2) * per_round
  Params prm;
  unsigned long long *acc;  // per frame: (pass-1 warp arrivals << 40) + sum of pEdge; zero on entry
  unsigned long long *sums; // per frame: S (written by the frame's first LUT task)
  double *means;            // per frame: S / (W H)
  float2 *luts;             // per frame: kLutSize entries {adj, osc}
  unsigned int *lut_done;   // per frame: finished LUT-task warps; zero on entry
  uint8_t *out;
  size_t out_pitch, out_fs;  // output bytes between rows / frames
  unsigned int *task_counter;  // zero on entry
  // kStepBandFused (kernels.h)
  unsigned long long *peer_slots[kMaxRanks];
  const unsigned long long *my_slots;
  unsigned long long epoch;
  int ranks;
  int halo_on, halo_bytes;
  unsigned long long *self_ctl, *up_ctl, *down_ctl;
  uint8_t *up_halo, *down_halo;
  const uint8_t *own_top, *own_bot;
};
// acc packing: S <= 1530 * W * H < 2^40 for W * H <= 2^29 (tma_supported),
// and the arrival count (4 per task) stays far below 2^24.
constexpr int kAccShift = 40;
template <bool kFused>
__device__ __forceinline__ int4 decode(const StepParams &sp, int t) {  // {type, frame, sub, 0}
  if (t >= sp.ntasks) return make_int4(kEnd, 0, 0, 0);
  // A row band's two launches (one frame): pass-1 tasks only; or the LUT
  // tasks (S preset by band_prep_kernel) followed by the pass-2 tasks.
  if (sp.mode == kStepPass1) return make_int4(kP1, 0, t, 0);
  if (sp.mode == kStepPass2) return t < kLutTasks ? make_int4(kLut, 0, t, 0) : make_int4(kP2, 0, t - kLutTasks, 0);
  if (kFused) {  // kStepBandFused: [halo push][pass 1][LUT][pass 2] of one band
    if (sp.halo_on) {
      if (t == 0) return make_int4(kHalo, 0, 0, 0);
      --t;
    }
    const int pf1 = sp.g.per_frame1;
    if (t < pf1) return make_int4(kP1, 0, t, 0);
    return t < pf1 + kLutTasks ? make_int4(kLut, 0, t - pf1, 0) : make_int4(kP2, 0, t - pf1 - kLutTasks, 0);
  }
  if (sp.compact) {  // a few frames: no lag rounds (their empty tasks cost a single image ~15 us)
    const int pf1 = sp.g.per_frame1, A = sp.n * pf1, B = A + sp.n * kLutTasks;
    if (t < A) return make_int4(kP1, t / pf1, t % pf1, 0);
    if (t < B) return make_int4(kLut, (t - A) / kLutTasks, (t - A) % kLutTasks, 0);
    return make_int4(kP2, (t - B) / sp.g.per_frame, (t - B) % sp.g.per_frame, 0);
  }
  const int rho = t / sp.per_round, k = t - rho * sp.per_round;
  const int pf1 = sp.g.per_frame1;
  if (k < pf1) return rho < sp.n ? make_int4(kP1, rho, k, 0) : make_int4(kEmpty, 0, 0, 0);
  if (k < pf1 + kLutTasks) {
    const int f = rho - sp.L1;
    return (f >= 0 && f < sp.n) ? make_int4(kLut, f, k - pf1, 0) : make_int4(kEmpty, 0, 0, 0);
  }
  const int f = rho - sp.L2;
  if (f < 0 || f >= sp.n) return make_int4(kEmpty, 0, 0, 0);
  return make_int4(kP2, f, k - pf1 - kLutTasks, 0);
}
__device__ __forceinline__ void tile_xy(const Geo &g, int sub, int th, int &C0, int &R0) {
  const int ty = sub / g.tiles_x;
  C0 = (sub - ty * g.tiles_x) * kCtaCols;
  R0 = g.row_lo + ty * th;
}
// ========================================================== pass 2, one row
// Output row of this lane (window rows a = r-1, b = r, c = r+1).
// V = vertical interpolation (x 128) of the four D columns (body, L146);
// D0 / D1 = 16*D of D rows r>>2 and (r>>2)+1 for the lane's D columns
// j0-1..j0+2 (border lines).  edge: 1 if the lane holds image columns 0,1,
// 2 if it holds W-2,W-1 (W % 16 == 0: only c0 == 0 / c0 == W-8), else 0.
template <bool kRingRows>
__device__ __forceinline__ void p2_row(const RowD &ra, const RowD &rb, const RowD &rc, const float4 &V,
                                       const float4 &D0, const float4 &D1, uint32_t lut_q,
                                       uint8_t *orow, uint64_t pol_out, bool store, int r, int c0, int W, int H,
                                       bool edge_warp, int edge, float cv, float dcv) {
  uint32_t pe[4], MX[4], MN[4];
  sobel(ra, rb, rc, pe);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    MX[i] = __vimax3_u16x2(ra.mx[i], rb.mx[i], rc.mx[i]);
    MN[i] = __vimin3_u16x2(ra.mn[i], rb.mn[i], rc.mn[i]);
  }
  // Upscale body (L146, R3), horizontal step on pixel pairs; NU = -U, exact.
  //   x = 0,1: (3,5),(1,7) on (V0,V1);  x = 2,3: (7,1),(5,3) on (V1,V2)
  //   x = 4,5: (3,5),(1,7) on (V1,V2);  x = 6,7: (7,1),(5,3) on (V2,V3)
  const float2 nu01 = lin2(V.x, V.y, cwt(0), cwt(1));
  const float2 nu23 = lin2(V.y, V.z, cwt(2), cwt(3));
  const float2 nu45 = lin2(V.y, V.z, cwt(0), cwt(1));
  const float2 nu67 = lin2(V.z, V.w, cwt(2), cwt(3));
  float NU[8] = {nu01.x, nu01.y, nu23.x, nu23.y, nu45.x, nu45.y, nu67.x, nu67.y};
  if (kRingRows && (r < 2 || r >= H - 2)) {  // warp-uniform
    ring_rows(NU, pe, MX, MN, D0, D1, r, c0, W, H, edge);
  } else if (edge_warp) {     // warp-uniform; only the edge lane changes
    // the column line's -U of this row (the third-last row takes the
    // fourth-last's, R4: one row step back; exact, multiples of 1/64)
    ring_cols_v(NU, pe, MX, MN, r == H - 3 ? __fsub_rn(cv, dcv) : cv, edge);
  }
  float P[8], T8[8], osc[8];
#pragma unroll
  for (int x = 0; x < 8; ++x) {
    const int p = pair_of(x);
    const bool hi = half_of(x);
    // f32 bits of 2^21 + pEdge = 0x4A000000 + 4 pEdge = 0x4A000000 + 8 k (ulp
    // 1/4; pEdge = 2k is even): the byte offset of entry k, scaled by the
    // exponent -- one FHADD, no IMAD.  (Even-only entries also spread the
    // lookups over all 32 banks.)
    const uint32_t q8 = __float_as_uint(add_f32_f16(hi ? hi16(pe[p]) : lo16(pe[p]), 2097152.0f));
    const float2 L = lds_f2(q8 + lut_q);  // {adj, osc}
    const float E = add_f32_f16(hi ? hi16(rb.c[p]) : lo16(rb.c[p]), NU[x]);                       // O - U (L148)
    P[x] = __fmaf_rn(L.x, E, -NU[x]);                                                              // L178
    const float mxf = add_f32_f16(hi ? hi16(MX[p]) : lo16(MX[p]), 0.0f);
    const float mnf = add_f32_f16(hi ? hi16(MN[p]) : lo16(MN[p]), 0.0f);
    T8[x] = fminf(fmaxf(P[x], mnf), mxf);  // Fig. 8 branch target (max / min / P)
    osc[x] = L.y;
  }
  float F[8];
#pragma unroll
  for (int x = 0; x < 8; x += 2) {
    const float2 d = sub2(make_float2(P[x], P[x + 1]), make_float2(T8[x], T8[x + 1]));
    F[x] = __fmaf_rn(osc[x], d.x, T8[x]);  // osc max / osc min / P
    F[x + 1] = __fmaf_rn(osc[x + 1], d.y, T8[x + 1]);
  }
  // clamp to [0, 255], RNE, pack (R14)
  const uint2 o = make_uint2(pack4_rni_u8(F[0], F[1], F[2], F[3]), pack4_rni_u8(F[4], F[5], F[6], F[7]));
  if (store) st_stream_u64(orow, o, pol_out);
}

using Ring = RingT<kStages, kStage>;

// Pass 2 of one warp over a task of nsub sub-tiles (stages s .. s+nsub-1,
// the first already waited for).  out: first row of the output rows
// [row_lo, row_hi).  Releases every stage it consumed.
// (Measured: a fully unrolled 12-row interior body -- no per-row phase or
// ring tests -- is 40% SLOWER: ~36 KB of straight-line code overflows the
// instruction cache.  The hot loops must stay small.)
__device__ __forceinline__ void p2_warp(const Ring &ring, int s, int nsub, uint32_t lut0, int lut_odd,
                                        uint8_t *__restrict__ out, uint32_t out_pitch,
                                        int W, int H, int row_lo, int row_hi, int C0w, int R0, int warp,
                                        int lane) {
  const int c0 = C0w + 8 * lane;
  const bool active = lane < 30 && c0 < W;
  // W % 8 == 0: image columns 0,1 are in the lane with c0 == 0, columns
  // W-2,W-1 in the lane with c0 == W-8.
  const int edge = !active ? 0 : (c0 == 0 ? 1 : (c0 == W - 8 ? 2 : 0));
  const bool edge_warp = (C0w == 0) || (C0w <= W - 8 && W - 8 < C0w + kTW);
  LR aw = lane_row_s(ring.stage(s), warp, lane);
  const uint64_t pol_out = policy_evict_first();  // output: written once, never re-read
  // LDS address of entry k = pEdge/2: the f32 bits of (2^21 + pEdge) plus
  // lut_q.  The vote makes the LUT-buffer choice -- and so lut_q -- provably
  // warp-uniform: ptxas keeps it in a uniform register and folds it into the
  // load, LDS [R + UR] (one FHADD + one LDS per pixel).
  const uint32_t lut_q = lut0 + (__any_sync(0xffffffffu, lut_odd) ? (uint32_t)kLutBytes : 0u) - 0x4A000000u;
  // In a sub-tile starting at row R0k, smem row of global row R0k-4 is 0:
  // row r -> smem row r - R0k + 4.
  // Vertical interpolation (L146, R3) of D rows (i, i+1) is linear in r on
  // r = 4i+2 .. 4i+5: V(r+1) = V(r) + 2 (D_{i+1} - D_i), restarted at
  // r = 4i+2 with V = 7 D_i + D_{i+1} (all exact integers, x 128).
  // State on entry to a sub-tile (rows R0k.., R0k % 4 == 0): D1 = D row
  // R0k/4 (the row-R0k update shifts it into D0 and loads the next), V and
  // slope of row R0k (a' = 0 of the interval (R0k/4 - 1, R0k/4): (3,5)).
  const float4 Dp = dblock(aw, 0, lane);  // D row R0/4 - 1
  float4 D1 = dblock(aw, 4, lane);        // D row R0/4
  float4 D0 = Dp;
  float4 V = f4fma(5.0f, D1, f4fma(3.0f, Dp, make_float4(0.f, 0.f, 0.f, 0.f)));
  float4 slope = f4twice_diff(D1, Dp);
  RowD ra = derive_w<true>(row_words(aw, 3), lane);
  RowD rb = derive_w<true>(row_words(aw, 4), lane);
  uint8_t *orow = out + (size_t)(R0 - row_lo) * out_pitch + c0;
  float cv = 0.0f, dcv = 0.0f;  // ring-column line: -U of the current row, and its row step (restarted at rr % 4 == 0)
#pragma unroll 1
  for (int k = 0; k < nsub; ++k) {
    const int R0k = R0 + k * kTH;
    if (k) {  // next sub-tile: same rows layout in the next stage; state carried
      ring.wait_full(s + k);
      aw = lane_row_s(ring.stage(s + k), warp, lane);
    }
    const int rend = min(R0k + kTH, row_hi);
    const int rend_l = active ? rend : R0k;  // this lane stores rows < rend_l
#pragma unroll 1
    for (int r = R0k; r < rend; r += 3) {
      // 3 rows per iteration: the window rotation has period 3, so the
      // unrolled body needs no register moves.
#pragma unroll
      for (int u = 0; u < 3; ++u) {
        const int rr = r + u;
        const int sm = rr - R0k + 4;
        if ((rr & 3) == 0) {  // next D block row
          D0 = D1;
          D1 = dblock(aw, sm + 4, lane);
          // Ring columns (L140-L142 steps ii/iv/vi): the column line of D
          // column 0 / w-1 between D rows rr/4 and rr/4 + 1 is linear in the
          // row: -U = -x0/16 - k (x1 - x0)/64 at row 4i + k, kept as cv += dcv
          // (exact: multiples of 1/64 below 256).
          const float x0 = edge == 1 ? D0.y : D0.z, x1 = edge == 1 ? D1.y : D1.z;
          cv = -div16(x0);
          dcv = __fmul_rn(__fsub_rn(x0, x1), 1.0f / 64.0f);
        } else if ((rr & 3) == 2) {  // next interpolation interval: D rows (k, k+1)
          V = f4fma(7.0f, D0, D1);
          slope = f4twice_diff(D1, D0);
        }
        const RowD rc = derive_w<true>(row_words(aw, sm + 1), lane);
        p2_row<true>(ra, rb, rc, V, D0, D1, lut_q, orow, pol_out, rr < rend_l, rr, c0, W, H, edge_warp, edge, cv, dcv);
        V = f4add(V, slope);
        cv = __fadd_rn(cv, dcv);
        orow += out_pitch;
        ra = rb;
        rb = rc;
      }
    }
    ring.release(s + k, lane);
  }
}

// ========================================================== pass 1 (warp)
// (Measured: a separate row-test-free loop for interior tiles, with or
// without pairwise f16 row sums, is no faster -- pass 1 waits on its TMA
// loads more than on issue -- and the 6-row variant's extra code is 5%
// slower.)
// Bytes are unpacked as f16 SUBNORMALS (derive_w<.., true>): every Sobel value
// is k * 2^-24 with |k| < 2048 exactly, and for such values the f16 BIT
// PATTERN is the integer k (subnormals, and the first normal binade whose
// spacing is still 2^-24).  pEdge <= 1530, so each f16x2 word of pe holds two
// pEdge values as u16 integers: the row sums are plain 32-bit integer adds of
// the words (each half stays < 2^16: <= 42 rows x 1530), two pixels per add,
// three rows per IADD3 pair; no conversions.
// One warp over a pass-1 task of nsub sub-tiles (stages s .. s+nsub-1, the
// first already waited for); releases every stage it consumed.
__device__ __forceinline__ uint32_t p1_warp(const Ring &ring, int s, int nsub, int warp, int W, int rmax1, int th1,
                                           int C0w, int R0, int lane) {
  const int c0 = C0w + 8 * lane;
  LR aw = lane_row_s(ring.stage(s), warp, lane);
  // smem row of global row R0-1 is 0: row r -> r - R0 + 1.
  RowD ra = derive_w<false, true>(row_words(aw, 0), lane);
  RowD rb = derive_w<false, true>(row_words(aw, 1), lane);
  uint32_t acc[4] = {0u, 0u, 0u, 0u};  // acc[i] = (sum of pEdge of pair i's low pixel, ... high pixel)
#pragma unroll 1
  for (int k = 0; k < nsub; ++k) {
    if (k) {  // next sub-tile: rows R0 + k th1 - 1 .. at smem row 0; the window (rows 0, 1) is carried
      ring.release(s + k - 1, lane);
      ring.wait_full(s + k);
      aw = lane_row_s(ring.stage(s + k), warp, lane);
      R0 += th1;
    }
    // rows 1 <= r <= rmax1 only (L160: the frame rows' pEdge is 0): decided
    // once per sub-tile (a vote: warp-uniform) -- every row valid is the
    // common case; only sub-tiles at the image's top / bottom test per row
    const bool all_rows = __all_sync(0xffffffffu, R0 >= 1 && R0 + th1 - 1 <= rmax1);
#pragma unroll 1
    for (int m = 0; m < th1; m += 3) {
      uint32_t pe[3][4];
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        const RowD rc = derive_w<false, true>(row_words(aw, m + a + 2), lane);
        sobel(ra, rb, rc, pe[a]);
        ra = rb;
        rb = rc;
      }
      const int r = R0 + m;
      if (all_rows) {
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
  }
  ring.release(s + nsub - 1, lane);
  // Sobel-body columns of this lane only (not the frame columns 0 / W-1, not
  // beyond the image, not the halo lanes): x = 4 (i >> 1) + (i & 1) + 2 half.
  uint32_t sum = 0;
  if (lane < 30) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int x = 4 * (i >> 1) + (i & 1);
      if (c0 + x >= 1 && c0 + x <= W - 2) sum += acc[i] & 0xffffu;
      if (c0 + x + 2 >= 1 && c0 + x + 2 <= W - 2) sum += acc[i] >> 16;
    }
  }
  return sum;
}

#ifdef SHARP_DIAG_TIMELINE  // timing experiment: globaltimer of the launch's phases (min / max over CTAs)
__device__ unsigned long long g_tl[8];
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define TL_MIN(i) atomicMin(&g_tl[i], gtimer())
#define TL_MAX(i) atomicMax(&g_tl[i], gtimer())
#else
#define TL_MIN(i)
#define TL_MAX(i)
#endif
// ============================================================== the kernel
// kFused: the one-band fused launch (kStepBandFused: in-kernel peer-memory
// all-reduce and halo push); a separate instantiation, so the batch kernel's
// code and registers are exactly those without it.
template <bool kFused>
__global__ void __launch_bounds__(kThreadsT, SHARP_LB_CTAS)
    step_kernel(const __grid_constant__ CUtensorMap map1A, const __grid_constant__ CUtensorMap map1B,
                const __grid_constant__ CUtensorMap map2A, const __grid_constant__ CUtensorMap map2B, StepParams sp) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ int4 stage_task[kStages];               // {type, frame, C0, R0} (LUT tasks: {type, frame, q, 0})
  __shared__ int2 stage_aux[kStages];                // pass 2: {sub-tiles of the task, LUT buffer}
  __shared__ unsigned long long stage_sum[kStages];  // LUT tasks: the frame's S
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t sbase = smem_u32(smem);
  const Ring ring{sbase, sbase + kBarOff, sbase + kBarOff + 8 * kStages};
  const uint32_t lutbase = sbase + kLutOff;
  const Geo &g = sp.g;

  if (threadIdx.x == 0) TL_MIN(0);
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(ring.full0 + 8 * i, 1);
      mbar_init(ring.empty0 + 8 * i, 32 * kWarpsT);  // every consumer thread arrives (RingT::release)
    }
    fence_barrier_init();
  }
  __syncthreads();

  if (warp == kWarpsT) {
    // ------------------------------------------------------------ producer
    if (lane != 0) return;
    const unsigned long long arrivals = (unsigned long long)(g.per_frame1 * kWarpsT) << kAccShift;
    const uint64_t pol_keep = policy_evict_last(), pol_drop = policy_evict_first();
    int t_next = (int)atomicAdd(sp.task_counter, 1u);
    // s: stages filled; j: pass-2 tasks (LUT buffer j & 1); lut_last0/1: the
    // last stage of the pass-2 task that used LUT buffer b.
    int lut_last0 = -kStages, lut_last1 = -kStages;  // (two scalars: no local-memory array)
    for (int s = 0, j = 0;;) {
      const int4 d = decode<kFused>(sp, t_next);
      // Resolve the task's dependency first (before waiting for a stage).
      unsigned long long S = 0;
      if (d.x == kLut) {
        // every pass-1 warp of the frame has added its partial (the global
        // barrier of L174's reduction)
        while (((S = ld_relaxed_u64(&sp.acc[d.y])) & ~((1ull << kAccShift) - 1)) != arrivals) __nanosleep(kPollNs);
        if (kFused) {
          // L174 across the bands: LUT task 0 publishes this band's partial
          // (epoch << 40 | S_g) into slot[rank] of every band's window; every
          // LUT task then sums the G slots of its own window once they all
          // carry the epoch (a dead peer traps after 10 s, not a hang).
          const unsigned long long mine = S & ((1ull << kAccShift) - 1), ep = sp.epoch & 0xffffffull;
          if (d.z == 0)
            for (int q = 0; q < sp.ranks; ++q) st_release_sys_u64(sp.peer_slots[q], (ep << 40) | mine);
          unsigned long long tot = 0;
          const unsigned long long t0 = gtime_ns();
          for (int q = 0; q < sp.ranks; ++q) {
            unsigned long long v;
            while (((v = ld_acquire_sys_u64(sp.my_slots + q)) >> 40) != ep) {
              __nanosleep(kPollNs);
              if (gtime_ns() - t0 > 10000000000ull) __trap();
            }
            tot += v & ((1ull << kAccShift) - 1);
          }
          S = tot;
        }
      }
      auto wait_sys = [&](const unsigned long long *p, unsigned long long want) {
        const unsigned long long t0 = gtime_ns();
        while (ld_acquire_sys_u64(p) != want) {
          __nanosleep(kPollNs);
          if (gtime_ns() - t0 > 10000000000ull) __trap();  // a dead peer: trap, not hang
        }
      };
      if (kFused && d.x == kHalo) {
        // (1) my previous launch is complete: the neighbours may fill my
        // halos of this epoch; (2) wait until they accept my edge rows
        if (sp.up_ctl) st_release_sys_u64(sp.up_ctl + kCtlReadyDown, sp.epoch);
        if (sp.down_ctl) st_release_sys_u64(sp.down_ctl + kCtlReadyUp, sp.epoch);
        if (sp.up_ctl) wait_sys(sp.self_ctl + kCtlReadyUp, sp.epoch);
        if (sp.down_ctl) wait_sys(sp.self_ctl + kCtlReadyDown, sp.epoch);
      }
      // (A pass-2 task's dependency -- its frame's LUT -- is resolved after
      // its first stage's tile loads are issued: the loads do not need it.)
      int C0 = 0, R0 = 0, nsub = 1, nw = 0;
      if (d.x == kP1 || d.x == kP2) {
        tile_xy(g, d.z, d.x == kP1 ? g.th1 * g.sub1 : kTH * g.sub, C0, R0);
        if (d.x == kP2) nsub = min(g.sub, (g.row_hi - R0 + kTH - 1) / kTH);
        if (d.x == kP1) nsub = min(g.sub1, (g.row_hi - R0 + g.th1 - 1) / g.th1);
#pragma unroll
        for (int w = 0; w < kWarpsT; ++w) nw += (C0 + w * kTW < g.W);
      }
      for (int k = 0; k < nsub; ++k, ++s) {
        const int b = Ring::buf(s);
        if (s >= kStages) mbar_wait(ring.empty0 + 8u * b, Ring::phase(s) ^ 1u);
        // Grab the following task while issuing this task's LAST stage: the
        // atomic's latency overlaps the stage's loads and the next empty-wait,
        // and the grabbed task starts about one task later (grabbing at the
        // first stage of a multi-stage task delayed it by the whole task, so
        // the dependency lags had to be 4x longer: 3.50 vs 2.23 B/px DRAM).
        if (k == nsub - 1 && d.x != kEnd) t_next = (int)atomicAdd(sp.task_counter, 1u);
        const uint32_t full = ring.full0 + 8u * b, st = ring.stage(s);
        if (d.x == kP1) {
          const int R0k = R0 + k * g.th1;
          if (kFused && sp.halo_on) {  // tiles at the band's edges read the neighbours' rows
            bool waited = false;
            if (sp.up_ctl && R0k == g.row_lo) {
              wait_sys(sp.self_ctl + kCtlDataUp, sp.epoch);
              waited = true;
            }
            if (sp.down_ctl && R0k + g.th1 >= g.row_hi) {
              wait_sys(sp.self_ctl + kCtlDataDown, sp.epoch);
              waited = true;
            }
            if (waited) fence_proxy_async_global();  // peer-written rows before the TMA reads them
          }
          stage_task[b] = make_int4(d.x, d.y, C0, R0k);  // consumers get the tile origin (no division there)
          stage_aux[b] = make_int2(nsub, 0);
          mbar_expect_tx(full, tile_bytes_s(nw, kRows1));
          tma_tiles_s(st, &map1A, &map1B, C0, nw, R0k - 1 - g.y0, d.y, full, pol_keep);
        } else if (d.x == kP2) {
          const int R0k = R0 + k * kTH;
          if (kFused && sp.halo_on) {  // (tile loads go out before the LUT wait: check the halo flags here too)
            bool waited = false;
            if (sp.up_ctl && R0k - 4 < g.row_lo) {
              wait_sys(sp.self_ctl + kCtlDataUp, sp.epoch);
              waited = true;
            }
            if (sp.down_ctl && R0k + kTH + 4 > g.row_hi) {
              wait_sys(sp.self_ctl + kCtlDataDown, sp.epoch);
              waited = true;
            }
            if (waited) fence_proxy_async_global();
          }
          stage_task[b] = make_int4(d.x, d.y, C0, R0k);
          stage_aux[b] = make_int2(nsub, j & 1);
          const uint32_t lut_bytes = k == 0 ? (uint32_t)kLutBytes : 0u;
          // LUT buffer j & 1 is free once the stages of pass-2 task j-2 are
          // released: stages <= s - kStages are (the empty wait above); a
          // later one only after single-stage pass-2 tasks.
          const int tl = (j & 1) ? lut_last1 : lut_last0;
          if (k == 0 && tl > s - kStages) mbar_wait(ring.empty0 + 8u * Ring::buf(tl), Ring::phase(tl));
          mbar_expect_tx(full, tile_bytes_s(nw, kRows2) + lut_bytes);
          // The frame's LUT (its LUT tasks were grabbed rounds earlier) is
          // normally complete: then the table copy goes out first.  Acquire
          // LOADS, not fence.acq_rel: a fence after this thread's tile loads
          // also waits for them (measured on the resident kernel: ~2 us).
          const unsigned want = (unsigned)(kLutTasks * kWarpsT);
          const bool lut_now = lut_bytes && ld_acquire(&sp.lut_done[d.y]) >= want;
          if (lut_now) {
            fence_proxy_async_global();
            bulk_copy(lutbase + (uint32_t)((j & 1) * kLutBytes), sp.luts + (size_t)d.y * kLutSize, kLutBytes, full);
          }
          tma_tiles_s(st, &map2A, &map2B, C0, nw, R0k - 4 - g.y0, d.y, full, pol_drop);
          if (lut_bytes && !lut_now) {
            while (ld_acquire(&sp.lut_done[d.y]) < want) __nanosleep(kPollNs);
            fence_proxy_async_global();
            bulk_copy(lutbase + (uint32_t)((j & 1) * kLutBytes), sp.luts + (size_t)d.y * kLutSize, kLutBytes, full);
          }
        } else {
          stage_task[b] = d;
          if (d.x == kLut) stage_sum[b] = S & ((1ull << kAccShift) - 1);
          // no data (LUT, empty or end task): a plain arrive publishes it
          mbar_arrive(full);
        }
      }
      if (d.x == kP2) {
        if (j & 1)
          lut_last1 = s - 1;
        else
          lut_last0 = s - 1;
        ++j;
      }
      if (d.x == kEnd) break;
    }
    return;
  }

  // -------------------------------------------------------------- consumers
  for (int s = 0;;) {
    const int b = Ring::buf(s);
    ring.wait_full(s);
    const int4 d = stage_task[b];
    if (d.x == kEnd) {
      if (lane == 0) TL_MAX(7);
      break;
    }
    if (d.x == kP2) {
      const int2 aux = stage_aux[b];
      const int C0 = d.z, R0 = d.w, C0w = C0 + warp * kTW;
      if (lane == 0) TL_MIN(5);
      if (C0w < g.W) {
        p2_warp(ring, s, aux.x, lutbase, aux.y, sp.out + (size_t)d.y * sp.out_fs, (uint32_t)sp.out_pitch, g.W, g.H,
                g.row_lo, g.row_hi, C0w, R0, warp, lane);
      } else {  // no columns for this warp: follow the stages
        for (int k = 0; k < aux.x; ++k) {
          if (k) ring.wait_full(s + k);
          ring.release(s + k, lane);
        }
      }
      if (lane == 0) TL_MAX(6);
      s += aux.x;
      continue;
    }
    if (d.x == kLut && lane == 0) TL_MIN(3);
    if (d.x == kP1 && lane == 0) TL_MIN(1);
    if (kFused && d.x == kHalo) {
      // push my first / last 4 rows into the neighbours' halos (16-byte peer
      // stores), make them visible system-wide, then flag them
      const int n16 = sp.halo_bytes / 16, tid = threadIdx.x;
      for (int i = tid; i < n16; i += kWarpsT * 32) {
        if (sp.up_halo) reinterpret_cast<uint4 *>(sp.up_halo)[i] = reinterpret_cast<const uint4 *>(sp.own_top)[i];
        if (sp.down_halo) reinterpret_cast<uint4 *>(sp.down_halo)[i] = reinterpret_cast<const uint4 *>(sp.own_bot)[i];
      }
      __threadfence_system();
      asm volatile("bar.sync 1, %0;" ::"n"(kWarpsT * 32) : "memory");  // the 4 consumer warps
      if (tid == 0) {
        if (sp.up_ctl) st_release_sys_u64(sp.up_ctl + kCtlDataDown, sp.epoch);
        if (sp.down_ctl) st_release_sys_u64(sp.down_ctl + kCtlDataUp, sp.epoch);
      }
    } else if (d.x == kLut) {
      // LUT task: entries k = q*128 .. q*128+127 (pEdge p = 2k) of frame f
      // (R9, R11; f64, one rounding).  (Measured: splitting adj / osc over two
      // threads per entry does not shorten the build and costs 0.9% of the batch.)
      const int f = d.y, k = d.z * kLutPerTask + threadIdx.x, p = 2 * k;
      // L174: mean of pEdge (R8), from the exact sum.
      const unsigned long long S = stage_sum[b];
      const double mean = frame_mean(S, g.W, g.H, sp.prm.flags);
      if (p == 0) {
        sp.sums[f] = S;
        sp.means[f] = mean;
      }
      sp.luts[(size_t)f * kLutSize + k] = p <= 1530 ? lut_entry(p, mean, sp.prm) : make_float2(0.0f, 0.0f);
      __threadfence();
      __syncwarp();
      if (lane == 0) atomicAdd(&sp.lut_done[f], 1u);
      if (lane == 0) TL_MAX(4);
    } else if (d.x == kP1) {
      const int C0 = d.z, R0 = d.w;
      const int C0w = C0 + warp * kTW;
      const int nsub = stage_aux[b].x;
      uint32_t acc = 0;
      if (C0w < g.W) {
        acc = p1_warp(ring, s, nsub, warp, g.W, g.rmax1, g.th1, C0w, R0, lane);
      } else {  // no columns for this warp: follow the stages
        for (int k = 0; k < nsub; ++k) {
          if (k) ring.wait_full(s + k);
          ring.release(s + k, lane);
        }
      }
      // Reduction (sec. V-C, Fig. 9): warp-shuffle reduction, then one u64
      // atomic per warp adding (1 << 40) + partial: the frame's arrival count
      // and sum in one word, so its LUT tasks can tell when S is complete
      // without any fence.
      const uint32_t ws = __reduce_add_sync(0xffffffffu, (uint32_t)acc);
      if (lane == 0) atomicAdd(&sp.acc[d.y], (1ull << kAccShift) + (unsigned long long)ws);
      if (lane == 0) TL_MAX(2);
      s += nsub;  // (p1_warp / the loop above released the task's stages)
      continue;
    }
    ring.release(s, lane);  // stage s may be refilled
    ++s;
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


// Per-device launch facts, filled by preload_step() (sharp_create calls it
// after selecting the context's device): SM count and the step kernel's
// resident CTAs per SM.  Atomics: contexts may be created from several threads.
constexpr int kMaxDevices = 64;
std::atomic<int> g_sms[kMaxDevices], g_resident[kMaxDevices];
int cur_device() {
  int dev = 0;
  cudaGetDevice(&dev);
  return (dev >= 0 && dev < kMaxDevices) ? dev : 0;
}
int num_sms() {
  const int v = g_sms[cur_device()].load(std::memory_order_relaxed);
  return v > 0 ? v : 148;
}

}  // namespace

#ifdef SHARP_DIAG_TIMELINE
extern "C" int sharp_debug_timeline(unsigned long long *out, int reset) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, g_tl, sizeof(g_tl));
  if (reset) {
    unsigned long long z[8];
    for (int i = 0; i < 8; ++i) z[i] = (i == 0 || i == 1 || i == 3 || i == 5) ? ~0ull : 0ull;
    cudaMemcpyToSymbol(g_tl, z, sizeof(z));
  }
  return 0;
}
#endif

bool make_map(CUtensorMap *m, const uint8_t *imgs, int n, int W, int H, size_t pitch, size_t fs, int box_cols,
              int box_rows) {
  auto fn = encode_fn();
  if (!fn) return false;
  const cuuint64_t dims[3] = {(cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)n};  // [n][H][W] at the given strides
  const cuuint64_t strides[2] = {(cuuint64_t)pitch, (cuuint64_t)fs};
  const cuuint32_t box[3] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows, 1};
  const cuuint32_t estr[3] = {1, 1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, (void *)imgs, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool tma_supported(const uint8_t *imgs, const uint8_t *outs, int W, int H) {
  return (W % 16) == 0 && tma_supported_strided(imgs, W, (size_t)W * H, outs, W, (size_t)W * H, W, H);
}

bool tma_supported_strided(const uint8_t *imgs, size_t in_pitch, size_t in_fs, const uint8_t *outs, size_t out_pitch,
                           size_t out_fs, int W, int H) {
  // (W >= 16: columns 0,1 and W-2,W-1 must sit in different lanes)
  return (W % 8) == 0 && W >= 16 && (((uintptr_t)imgs) & 15) == 0 && (in_pitch % 16) == 0 && (in_fs % 16) == 0 &&
         in_pitch >= (size_t)W && (((uintptr_t)outs) & 7) == 0 && (out_pitch % 8) == 0 && (out_fs % 8) == 0 &&
         out_pitch >= (size_t)W && H >= 8 && (size_t)W * H <= (1u << 29) && encode_fn() != nullptr;
}

// Row-band helpers (one thread): arm a band's pass-2 launch with the
// all-reduced S (arrival count complete, so the LUT tasks start at once), and
// export a band's pass-1 partial S.
__global__ void band_prep_kernel(unsigned long long *acc, unsigned int *lut_done, unsigned int *task_counter,
                                 const unsigned long long *total, unsigned long long arrivals) {
  acc[0] = arrivals | (total[0] & ((1ull << kAccShift) - 1));
  lut_done[0] = 0;
  task_counter[0] = 0;
}
__global__ void band_finish_kernel(const unsigned long long *acc, unsigned long long *partial) {
  partial[0] = acc[0] & ((1ull << kAccShift) - 1);
}

struct StepGeometry {
  int n, rows_in;               // tensor-map frames and rows
  int row_lo, row_hi, y0;       // rows processed; image row of map row 0
};

cudaError_t launch_step(const BatchLaunch &a, const StepGeometry &sg, int mode, int W, int H, const Params &p,
                        cudaStream_t stream) {
  if (sg.n <= 0 || sg.row_hi <= sg.row_lo) return cudaSuccess;
  CUtensorMap m1A, m1B, m2A, m2B;  // the same frames: pass-1 / pass-2 box heights, regions A / B
  const int R = sg.rows_in;
  const size_t ip = a.in_pitch ? a.in_pitch : (size_t)W, ifs = a.in_fs ? a.in_fs : ip * R;
  if (!make_map(&m1A, a.in, sg.n, W, R, ip, ifs, kPitch, kRows1) ||
      !make_map(&m1B, a.in, sg.n, W, R, ip, ifs, kPitchB, kRows1) ||
      !make_map(&m2A, a.in, sg.n, W, R, ip, ifs, kPitch, kRows2) ||
      !make_map(&m2B, a.in, sg.n, W, R, ip, ifs, kPitchB, kRows2))
    return cudaErrorInvalidValue;
  StepParams sp;
  sp.g.W = W;
  sp.g.H = H;
  sp.g.row_lo = sg.row_lo;
  sp.g.row_hi = sg.row_hi;
  sp.g.y0 = sg.y0;
  sp.g.rmax1 = std::min(H - 2, sg.row_hi - 1);
  const int rows = sg.row_hi - sg.row_lo;
  sp.g.tiles_x = (W + kCtaCols - 1) / kCtaCols;
  const int grid_ctas = kCtasPerSm * num_sms();
  // Latency: a launch with fewer kSub-row-group tasks than CTAs (one image,
  // a short batch, a small band) runs its pass 2 as single sub-tiles, 3x the
  // parallelism; big launches keep kSub (one LUT copy per kSub sub-tiles).
  const int per_frame_sub = sp.g.tiles_x * ((rows + kTH * kSub - 1) / (kTH * kSub));
  sp.g.sub = ((long long)sg.n * per_frame_sub < grid_ctas) ? 1 : kSub;
  // A single frame or two (compact schedule) are a few waves of tasks: take
  // kSub = 1 when its waves, counted in sub-tiles, are fewer (8K: 960 tasks on
  // 444 CTAs = 3 waves x 3 sub-tiles vs 2880 = 7 waves x 1: 74.3 -> 71.0 us;
  // 16K ties at 54 x 1 vs 18 x 3 and keeps kSub: sub = 1 measured 3% slower).
  if (sp.g.sub == kSub && sg.n < 4) {
    const long long t1 = (long long)sg.n * sp.g.tiles_x * ((rows + kTH - 1) / kTH);
    const long long ts = (long long)sg.n * per_frame_sub;
    if ((t1 + grid_ctas - 1) / grid_ctas < kSub * ((ts + grid_ctas - 1) / grid_ctas)) sp.g.sub = 1;
  }
  sp.g.per_frame = sp.g.tiles_x * ((rows + kTH * sp.g.sub - 1) / (kTH * sp.g.sub));
  // pass-1 tiles: as tall as kTH1 while the launch has >= one tile per CTA,
  // but not below 9 rows (3- and 6-row tiles are mostly warm-up rows and task
  // overhead: 512^2 17.6 -> 17.0 us, one 1080p 20.7 -> 19.0 us with 9)
  sp.g.th1 = kTH1;
#ifndef SHARP_MIN_TH1
#define SHARP_MIN_TH1 9
#endif
  while (sp.g.th1 > SHARP_MIN_TH1 && (long long)sg.n * sp.g.tiles_x * ((rows + sp.g.th1 - 1) / sp.g.th1) < grid_ctas)
    sp.g.th1 = sp.g.th1 == kTH1 ? 9 : sp.g.th1 - 3;
  // sub-tiles per pass-1 task: kSub1 while the launch keeps >= one task per CTA
  sp.g.sub1 = (sp.g.th1 == kTH1 &&
               (long long)sg.n * sp.g.tiles_x * ((rows + kSub1 * kTH1 - 1) / (kSub1 * kTH1)) >= grid_ctas)
                  ? kSub1
                  : 1;
  sp.g.per_frame1 = sp.g.tiles_x * ((rows + sp.g.th1 * sp.g.sub1 - 1) / (sp.g.th1 * sp.g.sub1));
  sp.mode = mode;
  sp.compact = 0;
  sp.n = sg.n;
  sp.per_round = sp.g.per_frame1 + kLutTasks + sp.g.per_frame;
#ifndef SHARP_GRID_CTAS
#define SHARP_GRID_CTAS kCtasPerSm
#endif
  const int resident = std::max(1, g_resident[cur_device()].load(std::memory_order_relaxed));
  int grid = std::min(SHARP_GRID_CTAS, resident) * num_sms();
  if (a.grid_cap > 0) grid = std::min(grid, a.grid_cap);
  if (mode == kStepPass1) {
    sp.L1 = sp.L2 = 0;
    sp.ntasks = sp.g.per_frame1;
  } else if (mode == kStepPass2) {
    sp.L1 = sp.L2 = 0;
    sp.ntasks = kLutTasks + sp.g.per_frame;
  } else if (mode == kStepBandFused) {
    sp.L1 = sp.L2 = 0;
    sp.ntasks = (a.halo_on ? 1 : 0) + sp.g.per_frame1 + kLutTasks + sp.g.per_frame;
  } else {
    // Lags (in rounds): a frame's LUT tasks come L1 rounds after its pass-1
    // tasks, its pass-2 tasks L2 rounds after them, so that dependencies are
    // normally complete when a producer checks them.  Reference distances:
    // the tasks the grid can hold (a current task and two stages per CTA)
    // before the LUT, and two grids' worth of grabs more before the pass 2.
    // A producer grabs its next task while it issues the current task's LAST
    // stage, so a grabbed task starts about one task after the grab, and half
    // of those distances suffice (measured, 1024 x 1080p: 0.5x 3.100 ms with
    // 2.23 B/px of DRAM traffic -- the frames stay in L2 for their pass 2 --
    // vs 1x 3.096 ms / 2.50 B/px; grabbing at the first stage needed 2x:
    // 3.15 ms / 3.50 B/px).  The lag rounds past the last frame hold only
    // empty tasks.  A dependency wait stalls one producer; it cannot
    // deadlock -- every dependency was grabbed, and issued, earlier.
#ifndef SHARP_LAG_X4
#define SHARP_LAG_X4 2  // lag multiplier x 4
#endif
    const int in_flight = 3 * grid;
    const int l1 = (in_flight + sp.per_round - 1) / sp.per_round + 1;
    const int l2 = l1 + std::max(1, (2 * grid + sp.per_round - 1) / sp.per_round);
    sp.L1 = std::max(1, l1 * SHARP_LAG_X4 / 4);
    sp.L2 = std::max(sp.L1 + 1, l2 * SHARP_LAG_X4 / 4);
    sp.ntasks = (sg.n + sp.L2) * sp.per_round;
    if (sg.n < kCompactN) {  // [pass 1 of all][LUT of all][pass 2 of all]: every dependency precedes its task
      sp.compact = 1;
      sp.ntasks = sg.n * sp.per_round;
    }
  }
  sp.prm = p;
  sp.acc = a.acc;
  sp.sums = a.sums;
  sp.means = a.means;
  sp.luts = a.luts;
  sp.lut_done = a.lut_done;
  for (int q = 0; q < kMaxRanks; ++q) sp.peer_slots[q] = a.peer_slots[q];
  sp.my_slots = a.my_slots;
  sp.epoch = a.epoch;
  sp.ranks = a.ranks;
  sp.halo_on = a.halo_on;
  sp.halo_bytes = a.halo_bytes;
  sp.self_ctl = a.self_ctl;
  sp.up_ctl = a.up_ctl;
  sp.down_ctl = a.down_ctl;
  sp.up_halo = a.up_halo;
  sp.down_halo = a.down_halo;
  sp.own_top = a.own_top;
  sp.own_bot = a.own_bot;
  sp.out = a.out;
  sp.out_pitch = a.out_pitch ? a.out_pitch : (size_t)W;
  sp.out_fs = a.out_fs ? a.out_fs : sp.out_pitch * (size_t)H;
  sp.task_counter = a.task_counter;
  if (mode == kStepPass2) {
    band_prep_kernel<<<1, 1, 0, stream>>>(a.acc, a.lut_done, a.task_counter, a.total,
                                          (unsigned long long)(sp.g.per_frame1 * kWarpsT) << kAccShift);
  }
  if (mode == kStepBandFused)
    step_kernel<true><<<grid, kThreadsT, kSmem, stream>>>(m1A, m1B, m2A, m2B, sp);
  else
    step_kernel<false><<<grid, kThreadsT, kSmem, stream>>>(m1A, m1B, m2A, m2B, sp);
  if (mode == kStepPass1) band_finish_kernel<<<1, 1, 0, stream>>>(a.acc, a.partial);
  return cudaGetLastError();
}

cudaError_t launch_batch_tma(const BatchLaunch &a, int W, int H, const Params &p, cudaStream_t stream) {
  return launch_step(a, StepGeometry{a.n, H, 0, H, 0}, kStepAll, W, H, p, stream);
}

cudaError_t launch_band_tma(const BatchLaunch &a, int mode, int W, int H, int row_lo, int row_hi, int y0, int rows_in,
                            const Params &p, cudaStream_t stream) {
  if (mode != kStepPass1 && mode != kStepPass2 && mode != kStepBandFused) return cudaErrorInvalidValue;
  return launch_step(a, StepGeometry{1, rows_in, row_lo, row_hi, y0}, mode, W, H, p, stream);
}

// Forces the (lazy) module load of this file's kernels; see kernels.h.
cudaError_t preload_step() {
  cudaFuncAttributes a;
  cudaError_t e;
  // the dynamic smem opt-in is a per-device function attribute: set it for
  // the current (the context's) device
  if ((e = cudaFuncSetAttribute(step_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem)) != cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(step_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem)) != cudaSuccess)
    return e;
  const int dev = cur_device();
  int sms = 0, res = 0;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&res, step_kernel<false>, kThreadsT, kSmem)) != cudaSuccess)
    return e;
  g_sms[dev].store(sms > 0 ? sms : 148);
  g_resident[dev].store(res > 0 ? res : 1);
  if ((e = cudaFuncGetAttributes(&a, step_kernel<false>)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, step_kernel<true>)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, band_prep_kernel)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, band_finish_kernel)) != cudaSuccess) return e;
  return cudaSuccess;
}

}  // namespace sharp
