/*
 * oracle/oracle.c -- CPU ORACLE (test infrastructure only; see oracle.h).
 *
 * Plain whole-image C, one stage at a time, in the order of PAPER.md
 * section III.  No tiling, no fusion, no lookup tables, nothing shared with
 * the CUDA path.  Compile: -O2 -ffp-contract=off (no fast-math).
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int oracle_check_geometry(int W, int H) {
  /* R1: 8-bit single channel, W x H, both multiples of 4 (the downscale
   * output is width/4 x height/4, L130) and at least 8 (two 4x4 blocks per
   * side, so the body upscale of L146 has at least one 2x2 window). */
  if (W < 8 || H < 8 || (W % 4) != 0 || (H % 4) != 0) return -1;
  return 0;
}

/* ---------------------------------------------------------------------------
 * Downscale, L130 + L136 (Fig. 2) + L218: "the value of an element in the
 * downscaled matrix is the mean value of the elements in the corresponding
 * 4 x 4 submatrix".  R2: exact mean (sum/16 is exact in float).
 * ------------------------------------------------------------------------- */
void oracle_downscale(const uint8_t *O, int W, int H, float *D) { oracle_downscale_ex(O, W, H, 0, D); }

/* flags & ORACLE_READ_INT_DOWNSCALE (R2 alternative, "shifts replace
 * division", L374): D = floor(sum / 16), the integer shift sum >> 4. */
void oracle_downscale_ex(const uint8_t *O, int W, int H, int flags, float *D) {
  const int w = W / 4, h = H / 4;
  for (int i = 0; i < h; ++i)
    for (int j = 0; j < w; ++j) {
      unsigned sum = 0;
      for (int a = 0; a < 4; ++a)
        for (int b = 0; b < 4; ++b) sum += O[(size_t)(4 * i + a) * W + (4 * j + b)];
      D[(size_t)i * w + j] = (flags & ORACLE_READ_INT_DOWNSCALE) ? (float)(sum >> 4) : (float)sum / 16.0f;
    }
}

/* ---------------------------------------------------------------------------
 * Upscale, L138-L146.
 *
 * Border (L140-L142, Fig. 3; readings R4, R5).  `line` places the downscaled
 * values every fourth element and fills the three vacancies between two of
 * them with the weights (3:1, 2:2, 1:3)/4 -- the "predefined parameter
 * matrix" applied to the two adjacent (red) values.  All elements except the
 * last three are computed that way; "the third last element's value is copied
 * from the fourth last value".  So line() writes out[0 .. n-3].
 * ------------------------------------------------------------------------- */
static double lerp_k(double x, double y, int k) { return ((4 - k) * x + k * y) / 4.0; }

/* v: n/4 values with stride `vs`; out: n-2 values written with stride `os`. */
static void line(const float *v, int vs, int n, float *out, int os) {
  for (int c = 0; c <= n - 4; ++c) {
    const int j = c >> 2, k = c & 3;
    const double val = (k == 0) ? (double)v[(size_t)j * vs]
                                : lerp_k(v[(size_t)j * vs], v[(size_t)(j + 1) * vs], k);
    out[(size_t)c * os] = (float)val;
  }
  out[(size_t)(n - 3) * os] = out[(size_t)(n - 4) * os]; /* third last <- fourth last */
}

void oracle_upscale(const float *D, int W, int H, float *U) { oracle_upscale_steps_ex(D, W, H, U, 8, 0); }

void oracle_upscale_steps(const float *D, int W, int H, float *U, int last_step) {
  oracle_upscale_steps_ex(D, W, H, U, last_step, 0);
}

void oracle_upscale_ex(const float *D, int W, int H, int flags, float *U) {
  oracle_upscale_steps_ex(D, W, H, U, 8, flags);
}

/* Default order: steps (i)..(vii) as L140-L142 list them (R5).  With
 * flags & ORACLE_READ_COLUMN_WINS (the R5 alternative) the row work comes
 * first -- (i), (iii), (v) -- and the column work after it -- (ii), (iv),
 * (vi) -- so in the top-left 2x2 the column line and the column copy are the
 * last writers; (vii) stays last.  last_step counts steps in the order run. */
void oracle_upscale_steps_ex(const float *D, int W, int H, float *U, int last_step, int flags) {
  const int w = W / 4, h = H / 4;
  static const int order_default[7] = {1, 2, 3, 4, 5, 6, 7};
  static const int order_colwins[7] = {1, 3, 5, 2, 4, 6, 7};
  const int *order = (flags & ORACLE_READ_COLUMN_WINS) ? order_colwins : order_default;
  /* Fill with NaN so a pixel that no step writes is visible (the pins check
   * that none is left). */
  for (size_t p = 0; p < (size_t)W * H; ++p) U[p] = NAN;
#define U_(r, c) U[(size_t)(r) * W + (c)]
#define D_(i, j) D[(size_t)(i) * w + (j)]

  /* 1) Upscale the border (L140-L142). */
  for (int k = 0; k < 7 && k < last_step; ++k) {
    switch (order[k]) {
      case 1: /* (i)  first row of D -> first row of U, columns 0..W-3 */
        line(&D_(0, 0), 1, W, &U_(0, 0), 1);
        break;
      case 2: /* (ii) first column of D -> first column of U, rows 0..H-3 */
        line(&D_(0, 0), w, H, &U_(0, 0), W);
        break;
      case 3: /* (iii) "the penultimate row ... based on the last row" of D */
        line(&D_(h - 1, 0), 1, W, &U_(H - 2, 0), 1);
        break;
      case 4: /* (iv) "the penultimate ... column ... based on the last ... column" of D */
        line(&D_(0, w - 1), w, H, &U_(0, W - 2), W);
        break;
      case 5: /* (v) "copied directly to the second row" / "copied to the last row"
               *     (over the columns the row passes computed, 0..W-3) */
        for (int c = 0; c <= W - 3; ++c) {
          U_(1, c) = U_(0, c);
          U_(H - 1, c) = U_(H - 2, c);
        }
        break;
      case 6: /* (vi) "... and column respectively" / "... and the last column"
               *      (over the rows the column passes computed, 0..H-3) */
        for (int r = 0; r <= H - 3; ++r) {
          U_(r, 1) = U_(r, 0);
          U_(r, W - 1) = U_(r, W - 2);
        }
        break;
      default: { /* (vii) "the four elements of the bottom right corner are still
                  * missing.  The third last value of the last column will be
                  * copied to those elements" */
        const float v = U_(H - 3, W - 1);
        U_(H - 2, W - 2) = v;
        U_(H - 2, W - 1) = v;
        U_(H - 1, W - 2) = v;
        U_(H - 1, W - 1) = v;
      }
    }
  }

  if (last_step < 8) return;
  /* 2) Upscale the main body (L146, Figs. 4-5): every stride-4 4x4 block of
   * U is P * Dsub * P^T with Dsub the stride-1 2x2 window of D and P the
   * predefined 4x2 parameter matrix (R3: half-pixel bilinear weights, blocks
   * at offset 2 so that body + 2-pixel border tile the image exactly). */
  static const double P[4][2] = {{7.0 / 8, 1.0 / 8},
                                 {5.0 / 8, 3.0 / 8},
                                 {3.0 / 8, 5.0 / 8},
                                 {1.0 / 8, 7.0 / 8}};
  for (int i = 0; i <= h - 2; ++i)
    for (int j = 0; j <= w - 2; ++j) {
      const double Dsub[2][2] = {{D_(i, j), D_(i, j + 1)}, {D_(i + 1, j), D_(i + 1, j + 1)}};
      double T[4][2]; /* T = P * Dsub */
      for (int a = 0; a < 4; ++a)
        for (int q = 0; q < 2; ++q) T[a][q] = P[a][0] * Dsub[0][q] + P[a][1] * Dsub[1][q];
      for (int a = 0; a < 4; ++a) /* block = T * P^T */
        for (int b = 0; b < 4; ++b)
          U_(4 * i + 2 + a, 4 * j + 2 + b) = (float)(T[a][0] * P[b][0] + T[a][1] * P[b][1]);
    }
#undef U_
#undef D_
}

/* ---------------------------------------------------------------------------
 * pError, L148: "the difference matrix between the upscaled matrix and the
 * original matrix".  R6: E = O - U (so that an adjusted pEdge of 1 gives back
 * the original, the unsharp-mask form).  Exact in float.
 * ------------------------------------------------------------------------- */
void oracle_perror(const uint8_t *O, const float *U, int n, float *E) {
  for (int p = 0; p < n; ++p) E[p] = (float)O[p] - U[p];
}

/* ---------------------------------------------------------------------------
 * Sobel, L158-L172 (Figs. 6-7).  a) border rows/cols = 0 (L160); b) body:
 * the pair of 3x3 Sobel masks on the 3x3 window centred on the element
 * (L164), result = |Gx| + |Gy| (L166).  R7: the standard (1,2,1) pair.
 * ------------------------------------------------------------------------- */
void oracle_sobel(const uint8_t *O, int W, int H, int32_t *pE) {
  static const int Mx[3][3] = {{-1, 0, 1}, {-2, 0, 2}, {-1, 0, 1}};
  static const int My[3][3] = {{-1, -2, -1}, {0, 0, 0}, {1, 2, 1}};
  for (int r = 0; r < H; ++r)
    for (int c = 0; c < W; ++c) {
      if (r == 0 || c == 0 || r == H - 1 || c == W - 1) {
        pE[(size_t)r * W + c] = 0;
        continue;
      }
      int gx = 0, gy = 0;
      for (int u = -1; u <= 1; ++u)
        for (int v = -1; v <= 1; ++v) {
          const int o = O[(size_t)(r + u) * W + (c + v)];
          gx += Mx[u + 1][v + 1] * o;
          gy += My[u + 1][v + 1] * o;
        }
      pE[(size_t)r * W + c] = abs(gx) + abs(gy);
    }
}

/* ---------------------------------------------------------------------------
 * Reduction, L174 ("the arithmetic mean of the elements in this matrix") and
 * L284 ("the sum of sobel matrix").  R8: all W*H elements (zero frame
 * included); exact u64 sum; mean in double.
 * ------------------------------------------------------------------------- */
void oracle_reduce(const int32_t *pE, int W, int H, uint64_t *S, double *mean) {
  oracle_reduce_ex(pE, W, H, 0, S, mean);
}

/* flags & ORACLE_READ_INTERIOR_MEAN (R8 alternative): the mean over the
 * (W-2)(H-2) body elements only (the frame is 0 either way, so S is equal). */
void oracle_reduce_ex(const int32_t *pE, int W, int H, int flags, uint64_t *S, double *mean) {
  uint64_t s = 0;
  for (size_t p = 0; p < (size_t)W * H; ++p) s += (uint64_t)pE[p];
  *S = s;
  if (flags & ORACLE_READ_INTERIOR_MEAN)
    *mean = (double)s / ((double)(W - 2) * (double)(H - 2));
  else
    *mean = (double)s / ((double)W * (double)H);
}

/* ---------------------------------------------------------------------------
 * Brightness strength, L178 + L232.  "From the mean value and user-defined
 * parameters, brightness strength will be worked out. It is used to adjust
 * the pEdge matrix" and the strength matrix "will perform many
 * exponentiations".  R9: adj = A * (pE / m)^gamma with m = max(mean, 1),
 * evaluated in double and rounded once to float.  pow(0, 0) = 1.
 * ------------------------------------------------------------------------- */
void oracle_strength(const int32_t *pE, int n, double mean, float A, float gamma,
                     float *adj) {
  oracle_strength_ex(pE, n, mean, A, gamma, 1.0f, 0, adj);
}

/* flags & ORACLE_READ_STRENGTH_EXP (R9 alternative, a saturating curve):
 * adj = A * (1 - exp(-pE / (K*m))), K = the osc_scale parameter. */
void oracle_strength_ex(const int32_t *pE, int n, double mean, float A, float gamma, float K,
                        int flags, float *adj) {
  const double m = mean > 1.0 ? mean : 1.0;
  for (int p = 0; p < n; ++p) {
    if (flags & ORACLE_READ_STRENGTH_EXP)
      adj[p] = (float)((double)A * (1.0 - exp(-(double)pE[p] / ((double)K * m))));
    else
      adj[p] = (float)((double)A * pow((double)pE[p] / m, (double)gamma));
  }
}

/* ---------------------------------------------------------------------------
 * Preliminary sharpened matrix, L178: "the adjusted pEdge matrix will be
 * multiplied by the pError matrix ... This multiplication result summed with
 * the upscaled matrix".  R10: one rounding (fmaf).
 * ------------------------------------------------------------------------- */
void oracle_preliminary(const float *adj, const float *E, const float *U, int n,
                        float *P) {
  for (int p = 0; p < n; ++p) P[p] = fmaf(adj[p], E[p], U[p]);
}

/* ---------------------------------------------------------------------------
 * Overshoot control, L180-L212 (Fig. 8).
 *  a) Matrix border (L208): first/last row and column copied from the
 *     preliminary matrix; R13: clamped to [0,255] so it fits the image.
 *  b) Matrix body (L210-L212): max/min of the 3x3 window of the ORIGINAL
 *     matrix (L182, "max and min value of the 3*3 units of the original
 *     matrix"); oscStrength of the pEdge (L184); Fig. 8 branches:
 *       P > max: Final = min(osc max, 255)
 *       P < min: Final = max(osc min, 0)
 *       else   : Final = min(max(P, 0), 255)
 *     R11: osc = clamp(G * exp(-pE / (K*m)), 0, 1) (double, rounded once);
 *          osc max = max + osc * (P - max), osc min = min + osc * (P - min)
 *          ("max value adjusted by user-defined tuning parameters and the
 *          difference of the element and max value", L210), single fmaf.
 * ------------------------------------------------------------------------- */
void oracle_overshoot(const uint8_t *O, const float *P, const int32_t *pE, int W,
                      int H, double mean, float G, float K, float *F) {
  oracle_overshoot_ex(O, P, pE, W, H, mean, G, K, 0, F);
}

/* flags & ORACLE_READ_OSC_CONST (R11 alternative): oscStrength = G for every
 * element (no dependence on pEdge). */
void oracle_overshoot_ex(const uint8_t *O, const float *P, const int32_t *pE, int W,
                         int H, double mean, float G, float K, int flags, float *F) {
  const double m = mean > 1.0 ? mean : 1.0;
  for (int r = 0; r < H; ++r)
    for (int c = 0; c < W; ++c) {
      const size_t p = (size_t)r * W + c;
      const float pre = P[p];
      if (r == 0 || c == 0 || r == H - 1 || c == W - 1) {
        F[p] = fminf(fmaxf(pre, 0.0f), 255.0f);
        continue;
      }
      int mx = 0, mn = 255;
      for (int u = -1; u <= 1; ++u)
        for (int v = -1; v <= 1; ++v) {
          const int o = O[(size_t)(r + u) * W + (c + v)];
          if (o > mx) mx = o;
          if (o < mn) mn = o;
        }
      const float fmx = (float)mx, fmn = (float)mn;
      const float osc =
          (flags & ORACLE_READ_OSC_CONST)
              ? G
              : (float)fmin(fmax((double)G * exp(-(double)pE[p] / ((double)K * m)), 0.0), 1.0);
      if (pre > fmx) {
        const float osc_max = fmaf(osc, pre - fmx, fmx);
        F[p] = fminf(osc_max, 255.0f);
      } else if (pre < fmn) {
        const float osc_min = fmaf(osc, pre - fmn, fmn);
        F[p] = fmaxf(osc_min, 0.0f);
      } else {
        F[p] = fminf(fmaxf(pre, 0.0f), 255.0f);
      }
    }
}

/* R14: round half to even (default FP environment) to 8 bits. */
void oracle_output(const float *F, int n, uint8_t *out) { oracle_output_ex(F, n, 0, out); }

/* flags & ORACLE_READ_TRUNCATE (R14 alternative): the C cast, truncation
 * toward zero (F is already in [0, 255]). */
void oracle_output_ex(const float *F, int n, int flags, uint8_t *out) {
  for (int p = 0; p < n; ++p)
    out[p] = (flags & ORACLE_READ_TRUNCATE) ? (uint8_t)truncf(F[p]) : (uint8_t)nearbyintf(F[p]);
}

static int params_ok(float A, float gamma, float G, float K) {
  /* DESIGN.md R16 ranges; NaN fails every comparison. */
  if (!(A >= 0.0f && A <= 16.0f)) return 0;
  if (!(gamma >= 0.0f && gamma <= 4.0f)) return 0;
  if (!(G >= 0.0f && G <= 1.0f)) return 0;
  if (!(K > 0.0f && K <= 1.0e6f)) return 0;
  return 1;
}

/* The pipeline on a W x H image with W, H multiples of 4 (R1), stages in the
 * order of Fig. 1, each with the reading switches of `flags`. */
static int sharpen_core(const uint8_t *O, int W, int H, float A, float gamma, float G, float K, int flags,
                        uint8_t *out, uint64_t *S_out, double *mean_out) {
  const size_t n = (size_t)W * H;
  float *D = (float *)malloc(sizeof(float) * (n / 16));
  float *U = (float *)malloc(sizeof(float) * n);
  float *E = (float *)malloc(sizeof(float) * n);
  int32_t *pE = (int32_t *)malloc(sizeof(int32_t) * n);
  float *adj = (float *)malloc(sizeof(float) * n);
  float *P = (float *)malloc(sizeof(float) * n);
  float *F = (float *)malloc(sizeof(float) * n);
  int rc = -1;
  if (D && U && E && pE && adj && P && F) {
    uint64_t S;
    double mean;
    oracle_downscale_ex(O, W, H, flags, D);    /* Fig. 1: downscale()  */
    oracle_upscale_ex(D, W, H, flags, U);      /* Fig. 1: upscale()    */
    oracle_perror(O, U, (int)n, E);            /* Fig. 1: pError()     */
    oracle_sobel(O, W, H, pE);                 /* Fig. 1: Sharpness(): */
    oracle_reduce_ex(pE, W, H, flags, &S, &mean);                 /* Sobel, reduction, */
    oracle_strength_ex(pE, (int)n, mean, A, gamma, K, flags, adj); /* strength,         */
    oracle_preliminary(adj, E, U, (int)n, P);                     /* preliminary,      */
    oracle_overshoot_ex(O, P, pE, W, H, mean, G, K, flags, F);    /* overshoot         */
    oracle_output_ex(F, (int)n, flags, out);
    if (S_out) *S_out = S;
    if (mean_out) *mean_out = mean;
    rc = 0;
  }
  free(D); free(U); free(E); free(pE); free(adj); free(P); free(F);
  return rc;
}

int oracle_sharpen(const uint8_t *O, int W, int H, float A, float gamma, float G,
                   float K, uint8_t *out, uint64_t *S_out, double *mean_out) {
  if (oracle_check_geometry(W, H) != 0 || !params_ok(A, gamma, G, K)) return -1;
  return sharpen_core(O, W, H, A, gamma, G, K, 0, out, S_out, mean_out);
}

/* General geometry (reading R1' in DESIGN.md):
 * any W, H >= 5.  The image is extended to W4 x H4 (the next multiples of 4)
 * by replicating its last column and last row, the pipeline runs on the
 * extended image (so S and the mean are those of the extended image), and the
 * output is its top-left W x H.  For W, H multiples of 4 this is exactly
 * oracle_sharpen.  Rows are read / written with the given pitches (bytes). */
int oracle_sharpen_ex(const uint8_t *O, int W, int H, int in_pitch, float A, float gamma, float G, float K,
                      int flags, uint8_t *out, int out_pitch, uint64_t *S_out, double *mean_out) {
  if (W < 5 || H < 5 || in_pitch < W || out_pitch < W || !params_ok(A, gamma, G, K)) return -1;
  if (flags & ~ORACLE_READ_ALL) return -1;
  const int W4 = (W + 3) / 4 * 4, H4 = (H + 3) / 4 * 4;
  uint8_t *X = (uint8_t *)malloc((size_t)W4 * H4);
  uint8_t *Y = (uint8_t *)malloc((size_t)W4 * H4);
  int rc = -1;
  if (X && Y) {
    for (int r = 0; r < H4; ++r)
      for (int c = 0; c < W4; ++c)
        X[(size_t)r * W4 + c] = O[(size_t)(r < H ? r : H - 1) * in_pitch + (c < W ? c : W - 1)];
    rc = sharpen_core(X, W4, H4, A, gamma, G, K, flags, Y, S_out, mean_out);
    if (rc == 0)
      for (int r = 0; r < H; ++r) memcpy(out + (size_t)r * out_pitch, Y + (size_t)r * W4, (size_t)W);
  }
  free(X);
  free(Y);
  return rc;
}

int oracle_sharpen_batch(const uint8_t *imgs, int n, int W, int H, float A,
                         float gamma, float G, float K, uint8_t *outs,
                         uint64_t *sums, int threads) {
  if (n < 1) return -1;
  int rc = 0;
  const size_t fs = (size_t)W * H;
#ifdef _OPENMP
  if (threads <= 0) threads = omp_get_max_threads();
#pragma omp parallel for num_threads(threads) schedule(dynamic, 1) reduction(| : rc)
#endif
  for (int f = 0; f < n; ++f) {
    uint64_t S = 0;
    rc |= oracle_sharpen(imgs + f * fs, W, H, A, gamma, G, K, outs + f * fs, &S, NULL);
    if (sums) sums[f] = S;
  }
  (void)threads;
  return rc ? -1 : 0;
}
