/*
 * synth/synth.c -- seeded synthetic 8-bit grayscale frames.
 *
 * Shared by the tests (oracle side and CUDA side get the same bytes) and by
 * bench.py.  It holds NONE of the sharpening method's arithmetic: it only
 * makes images.  Integer-only (splitmix64 hashing), so every platform
 * produces identical bytes for a given (kind, seed, frame, W, H, param).
 *
 * The paper's workloads are square 8-bit images 256^2..4096^2 (8192^2 in
 * Fig. 14) of unstated content.  Kinds:
 *   0 natural : smooth field (bilinear over a hashed 64-px grid) + 8..32
 *               hard-edged rectangles / discs (steps of +-40..120) +
 *               hashed noise in [-6, 6]; clamped to [0,255].  Exercises all
 *               three Fig. 8 overshoot branches.
 *   1 noise   : uniform u8 (worst case for branches / LUT locality).
 *   2 ramp    : piecewise-affine, slopes in {-1,0,1} per 64x64 tile.
 *   3 const   : every pixel = param.
 *   4 checker : 1-pixel checkerboard of (param, 255-param).
 *   5 impulse : zero image with 1..8 hashed impulses of height param, >=2 px
 *               away from the frame and >=5 px apart in Chebyshev distance.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static uint64_t mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static uint64_t h4(uint64_t seed, uint64_t a, uint64_t b, uint64_t c) {
  return mix(seed ^ mix(a * 0xD6E8FEB86659FD93ull ^ mix(b * 0xA0761D6478BD642Full ^ mix(c))));
}
static int clamp255(int v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

static void gen_natural(uint8_t *o, int W, int H, uint64_t s) {
  const int G = 64;
  const int gw = W / G + 2, gh = H / G + 2;
  int *grid = (int *)malloc(sizeof(int) * (size_t)gw * gh);
  int *acc = (int *)malloc(sizeof(int) * (size_t)W * H);
  for (int y = 0; y < gh; ++y)
    for (int x = 0; x < gw; ++x) grid[y * gw + x] = 40 + (int)(h4(s, 1, y, x) % 176);
  for (int r = 0; r < H; ++r) {
    const int gy = r / G, fy = r % G;
    for (int c = 0; c < W; ++c) {
      const int gx = c / G, fx = c % G;
      const int g00 = grid[gy * gw + gx], g01 = grid[gy * gw + gx + 1];
      const int g10 = grid[(gy + 1) * gw + gx], g11 = grid[(gy + 1) * gw + gx + 1];
      const int top = g00 * (G - fx) + g01 * fx, bot = g10 * (G - fx) + g11 * fx;
      const int noise = (int)(h4(s, 2, r, c) % 13) - 6;
      acc[(size_t)r * W + c] = ((top * (G - fy) + bot * fy) >> 12) + noise;
    }
  }
  const int nshapes = 8 + (int)(h4(s, 3, 0, 0) % 25);
  for (int k = 0; k < nshapes; ++k) {
    const uint64_t a = h4(s, 4, k, 0), b = h4(s, 5, k, 0);
    const int cy = (int)(a % (uint64_t)H), cx = (int)((a >> 32) % (uint64_t)W);
    int maxr = (W < H ? W : H) / 6;
    if (maxr < 3) maxr = 3;
    const int ry = 2 + (int)(b % (uint64_t)maxr), rx = 2 + (int)((b >> 20) % (uint64_t)maxr);
    int step = 40 + (int)((b >> 40) % 81);
    if ((b >> 60) & 1) step = -step;
    const int disc = (int)((b >> 61) & 1);
    const int y0 = cy - ry < 0 ? 0 : cy - ry, y1 = cy + ry >= H ? H - 1 : cy + ry;
    const int x0 = cx - rx < 0 ? 0 : cx - rx, x1 = cx + rx >= W ? W - 1 : cx + rx;
    for (int r = y0; r <= y1; ++r)
      for (int c = x0; c <= x1; ++c) {
        if (disc) {
          const int64_t dy = r - cy, dx = c - cx;
          if (dy * dy * (int64_t)rx * rx + dx * dx * (int64_t)ry * ry >
              (int64_t)rx * rx * (int64_t)ry * ry)
            continue;
        }
        acc[(size_t)r * W + c] += step;
      }
  }
  for (size_t p = 0; p < (size_t)W * H; ++p) o[p] = (uint8_t)clamp255(acc[p]);
  free(acc);
  free(grid);
}

static void gen_frame(uint8_t *o, int W, int H, int kind, uint64_t s, int param) {
  switch (kind) {
    case 0: gen_natural(o, W, H, s); break;
    case 1:
      for (int r = 0; r < H; ++r)
        for (int c = 0; c < W; ++c) o[(size_t)r * W + c] = (uint8_t)(h4(s, 6, r, c) & 255);
      break;
    case 2:
      for (int r = 0; r < H; ++r)
        for (int c = 0; c < W; ++c) {
          const uint64_t t = h4(s, 7, r / 64, c / 64);
          const int base = 64 + (int)(t % 128);
          const int bx = (int)((t >> 16) % 3) - 1, by = (int)((t >> 24) % 3) - 1;
          o[(size_t)r * W + c] = (uint8_t)clamp255(base + bx * (c % 64) + by * (r % 64));
        }
      break;
    case 3: memset(o, clamp255(param), (size_t)W * H); break;
    case 4:
      for (int r = 0; r < H; ++r)
        for (int c = 0; c < W; ++c)
          o[(size_t)r * W + c] = (uint8_t)(((r + c) & 1) ? clamp255(param) : 255 - clamp255(param));
      break;
    case 5: {
      memset(o, 0, (size_t)W * H);
      const int n = 1 + (int)(h4(s, 8, 0, 0) % 8);
      int placed = 0;
      for (int k = 0; k < 64 && placed < n; ++k) {
        const uint64_t a = h4(s, 9, k, 0);
        const int r = 2 + (int)(a % (uint64_t)(H - 4)), c = 2 + (int)((a >> 32) % (uint64_t)(W - 4));
        int ok = 1;
        for (int dr = -4; dr <= 4 && ok; ++dr)
          for (int dc = -4; dc <= 4 && ok; ++dc) {
            const int rr = r + dr, cc = c + dc;
            if (rr >= 0 && rr < H && cc >= 0 && cc < W && o[(size_t)rr * W + cc]) ok = 0;
          }
        if (!ok) continue;
        o[(size_t)r * W + c] = (uint8_t)clamp255(param);
        ++placed;
      }
      break;
    }
    default: memset(o, 0, (size_t)W * H);
  }
}

/* n frames [n][H][W]; frame f uses seed + f.  Returns 0 or -1. */
int synth_frames(uint8_t *dst, int n, int W, int H, int kind, uint64_t seed, int param,
                 int threads) {
  if (!dst || n < 1 || W < 8 || H < 8 || kind < 0 || kind > 5) return -1;
  const size_t fs = (size_t)W * H;
#ifdef _OPENMP
  if (threads <= 0) threads = omp_get_max_threads();
#pragma omp parallel for num_threads(threads) schedule(dynamic, 1)
#endif
  for (int f = 0; f < n; ++f) gen_frame(dst + f * fs, W, H, kind, seed + (uint64_t)f, param);
  (void)threads;
  return 0;
}
