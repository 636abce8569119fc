/*
 * oracle/oracle.h -- CPU ORACLE for the sharpness pipeline of
 *   M. Fan, H. Jia, Y. Zhang, X. An, T. Cao, "Optimizing Image Sharpening
 *   Algorithm on GPU", ICPP 2015  (section III).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_icpp_fanjzac15_b200/) never links, loads or
 * calls it, and this code shares nothing with the CUDA path (no headers,
 * no tables, no helpers).
 *
 * Plain, slow, whole-image, one stage after another, in the paper's order:
 *   downscale (L130) -> upscale border (L140-L142) -> upscale body (L146)
 *   -> pError (L148) -> Sobel (L158-L172) -> mean (L174)
 *   -> strength / adjusted pEdge (L178) -> preliminary (L178)
 *   -> overshoot control (L180-L212, Fig. 8) -> 8-bit output.
 * Every stage materialises its full matrix.  The readings of the places where
 * the paper is silent or garbled (R1..R16) are listed in DESIGN.md section 3;
 * each function below names the readings it relies on.
 *
 * Precision (R15): D, U and pError are dyadic rationals with small
 * numerators and are EXACT in float; the two transcendental per-pixel factors
 * are evaluated in double and rounded once to float; the preliminary value and
 * the overshoot chain -- the values that decide the integer output -- are f32
 * with explicit single-rounding fmaf, i.e. the decision is taken in the same
 * (f32) precision as the kernel (task rule: decisions in the kernel's
 * precision).  Build with -ffp-contract=off, no fast-math.
 *
 * Parity pins: every function is pinned by tests/test_oracle_pins.py against
 * closed forms, brute force, paper statements or a rational-arithmetic
 * evaluation.  The two functional forms that the paper does not print
 * (R9 strength curve, R11 oscStrength curve) are "parity unpinned" as to
 * their SHAPE: only their special cases are pinned.
 */
#ifndef SHARP_ORACLE_H
#define SHARP_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* R1: W, H multiples of 4 and >= 8.  Returns 0 if valid, -1 otherwise. */
int oracle_check_geometry(int W, int H);

/* L130/L136/L218: D[i][j] = mean of the 4x4 block O[4i..4i+3][4j..4j+3].
 * O: H*W bytes row-major.  D: (H/4)*(W/4) floats row-major. (R2) */
void oracle_downscale(const uint8_t *O, int W, int H, float *D);

/* L140-L142 (border, steps i..vii) then L146 (body, P*Dsub*P^T).
 * D: (H/4)*(W/4).  U: H*W floats.  (R3, R4, R5) */
void oracle_upscale(const float *D, int W, int H, float *U);
/* The same, stopping after step `last_step` (1..7 = border steps i..vii,
 * 8 = body, i.e. everything); unwritten pixels are NaN.  Lets the tests check
 * L142's statement that only the bottom-right 2x2 is missing after (vi). */
void oracle_upscale_steps(const float *D, int W, int H, float *U, int last_step);

/* L148: pError E = O - U  (R6).  n = W*H. */
void oracle_perror(const uint8_t *O, const float *U, int n, float *E);

/* L158-L172: pEdge; frame = 0, body = |Gx|+|Gy| of the 3x3 Sobel pair (R7). */
void oracle_sobel(const uint8_t *O, int W, int H, int32_t *pE);

/* L174: S = sum of all W*H pEdge elements (u64), mean = S / (W*H) (R8). */
void oracle_reduce(const int32_t *pE, int W, int H, uint64_t *S, double *mean);

/* L178 (+L232): adjusted pEdge adj = (float)(A * pow(pE/m, gamma)),
 * m = max(mean, 1)  (R9). */
void oracle_strength(const int32_t *pE, int n, double mean, float A, float gamma,
                     float *adj);

/* L178: preliminary P = fmaf(adj, E, U)  (R10). */
void oracle_preliminary(const float *adj, const float *E, const float *U, int n,
                        float *P);

/* L180-L212, Fig. 8: overshoot control -> final F in [0,255] (R11, R12, R13). */
void oracle_overshoot(const uint8_t *O, const float *P, const int32_t *pE, int W,
                      int H, double mean, float G, float K, float *F);

/* R14: out = round-half-even(F). */
void oracle_output(const float *F, int n, uint8_t *out);

/* The whole pipeline, stages in the order above.  Returns 0, or -1 on bad
 * geometry (R1) / parameters / allocation failure.  S and mean may be NULL. */
int oracle_sharpen(const uint8_t *O, int W, int H, float A, float gamma, float G,
                   float K, uint8_t *out, uint64_t *S, double *mean);

/* ---- Reading switches: the
 * alternative readings of places where the paper is silent, as flags of the
 * _ex functions (0 = the default readings above). */
#define ORACLE_READ_INT_DOWNSCALE 1  /* R2:  D = floor(block sum / 16) (integer shift, L374)   */
#define ORACLE_READ_COLUMN_WINS 2    /* R5:  border steps (i),(iii),(v),(ii),(iv),(vi),(vii)    */
#define ORACLE_READ_INTERIOR_MEAN 4  /* R8:  mean = S / ((W-2)(H-2))                            */
#define ORACLE_READ_STRENGTH_EXP 8   /* R9:  adj = A (1 - exp(-pE / (K m)))                     */
#define ORACLE_READ_OSC_CONST 16     /* R11: oscStrength = G                                    */
#define ORACLE_READ_TRUNCATE 32      /* R14: out = trunc(F)                                     */
#define ORACLE_READ_ALL 63
void oracle_downscale_ex(const uint8_t *O, int W, int H, int flags, float *D);
void oracle_upscale_ex(const float *D, int W, int H, int flags, float *U);
void oracle_upscale_steps_ex(const float *D, int W, int H, float *U, int last_step, int flags);
void oracle_reduce_ex(const int32_t *pE, int W, int H, int flags, uint64_t *S, double *mean);
void oracle_strength_ex(const int32_t *pE, int n, double mean, float A, float gamma, float K,
                        int flags, float *adj);
void oracle_overshoot_ex(const uint8_t *O, const float *P, const int32_t *pE, int W,
                         int H, double mean, float G, float K, int flags, float *F);
void oracle_output_ex(const float *F, int n, int flags, uint8_t *out);

/* General geometry (reading R1'): any W, H >= 5,
 * rows at in_pitch / out_pitch bytes.  The image is extended to the next
 * multiples of 4 by replicating the last column and row, sharpened (with the
 * reading switches `flags`), and cropped back to W x H; S / mean are those of
 * the extended image.  Returns 0, or -1 on bad arguments. */
int oracle_sharpen_ex(const uint8_t *O, int W, int H, int in_pitch, float A, float gamma, float G, float K,
                      int flags, uint8_t *out, int out_pitch, uint64_t *S, double *mean);

/* n frames [n][H][W], each exactly oracle_sharpen; frames split over
 * `threads` OpenMP threads (<=0: all).  sums may be NULL. */
int oracle_sharpen_batch(const uint8_t *imgs, int n, int W, int H, float A,
                         float gamma, float G, float K, uint8_t *outs,
                         uint64_t *sums, int threads);

#ifdef __cplusplus
}
#endif
#endif
