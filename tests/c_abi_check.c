/*
 * tests/c_abi_check.c -- the C ABI of include/sharp.h used from plain C (no
 * Python, no torch): device-resident and host (pageable) calls, a batch, the
 * general-layout entry point with an odd size and a reading switch, and the
 * error contract.  Every output is compared byte for byte with the CPU oracle
 * (test infrastructure: tests may link oracle/), inputs from synth/.
 *
 * Built by `make tests/c_abi_check`; run by tests/test_gpu_c_abi.py.  Prints
 * "c_abi_check ok" and exits 0 on success.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "../oracle/oracle.h"
#include "sharp.h"

int synth_frames(uint8_t *dst, int n, int W, int H, int kind, uint64_t seed, int param, int threads);

#define CHECK(cond, ...)                                   \
  do {                                                     \
    if (!(cond)) {                                         \
      fprintf(stderr, "c_abi_check FAILED: " __VA_ARGS__); \
      fprintf(stderr, "\n");                               \
      exit(1);                                             \
    }                                                      \
  } while (0)

static void compare(const uint8_t *got, const uint8_t *ref, size_t n, const char *what) {
  size_t bad = 0;
  for (size_t i = 0; i < n; ++i) bad += got[i] != ref[i];
  CHECK(bad == 0, "%s: %zu of %zu bytes differ from the oracle", what, bad, n);
}

int main(void) {
  sharp_ctx *ctx = NULL;
  CHECK(sharp_create(&ctx, NULL) == SHARP_OK, "sharp_create");
  sharp_params p;
  sharp_default_params(&p);
  p.amount = 2.0f;

  /* 1. one 1920x1080 image, device-resident (sharp_run) */
  {
    const int W = 1920, H = 1080;
    const size_t n = (size_t)W * H;
    uint8_t *img = malloc(n), *ref = malloc(n), *got = malloc(n);
    synth_frames(img, 1, W, H, 0, 0x5EED2015ull + 1, 0, 0);
    uint64_t S_ref = 0;
    double m_ref = 0.0;
    CHECK(oracle_sharpen(img, W, H, p.amount, p.gamma, p.osc_gain, p.osc_scale, ref, &S_ref, &m_ref) == 0, "oracle");
    uint8_t *d_in = NULL, *d_out = NULL;
    CHECK(cudaMalloc((void **)&d_in, n) == cudaSuccess && cudaMalloc((void **)&d_out, n) == cudaSuccess, "cudaMalloc");
    CHECK(cudaMemcpy(d_in, img, n, cudaMemcpyHostToDevice) == cudaSuccess, "H2D");
    CHECK(sharp_run(ctx, d_in, W, H, &p, d_out) == SHARP_OK, "sharp_run (device): %s", sharp_last_error(ctx));
    CHECK(cudaMemcpy(got, d_out, n, cudaMemcpyDeviceToHost) == cudaSuccess, "D2H");
    compare(got, ref, n, "sharp_run device 1080p");
    sharp_stats st;
    CHECK(sharp_get_stats(ctx, &st) == SHARP_OK && st.edge_sum == S_ref && st.edge_mean == m_ref, "stats S / mean");
    /* 2. the same image from pageable host memory */
    memset(got, 0, n);
    CHECK(sharp_run(ctx, img, W, H, &p, got) == SHARP_OK, "sharp_run (host)");
    compare(got, ref, n, "sharp_run host 1080p");
    cudaFree(d_in);
    cudaFree(d_out);
    free(img);
    free(ref);
    free(got);
  }

  /* 3. a batch of 5 frames 256x64 from host memory (sharp_run_batch) */
  {
    const int W = 256, H = 64, N = 5;
    const size_t fb = (size_t)W * H;
    uint8_t *imgs = malloc(N * fb), *ref = malloc(N * fb), *got = malloc(N * fb);
    synth_frames(imgs, N, W, H, 0, 0x5EED2015ull + 7, 0, 0);
    uint64_t sums[5];
    CHECK(oracle_sharpen_batch(imgs, N, W, H, p.amount, p.gamma, p.osc_gain, p.osc_scale, ref, sums, 0) == 0,
          "oracle batch");
    CHECK(sharp_run_batch(ctx, imgs, N, W, H, &p, got) == SHARP_OK, "sharp_run_batch");
    compare(got, ref, N * fb, "sharp_run_batch");
    uint64_t gsums[5];
    CHECK(sharp_get_batch_sums(ctx, gsums, N) == SHARP_OK, "batch sums");
    for (int f = 0; f < N; ++f) CHECK(gsums[f] == sums[f], "S of frame %d", f);
    free(imgs);
    free(ref);
    free(got);
  }

  /* 4. sharp_run_ex: a 333x77 region of interest (row pitch 400) with the R14
   *    truncation switch, written into a pitched output */
  {
    const int W = 333, H = 77, PITCH = 400;
    uint8_t *big = malloc((size_t)PITCH * H), *ref = malloc((size_t)W * H), *out = malloc((size_t)PITCH * H);
    synth_frames(big, 1, PITCH, H, 0, 0x5EED2015ull + 9, 0, 0);
    memset(out, 0xAB, (size_t)PITCH * H);
    uint64_t S_ref = 0;
    double m_ref = 0.0;
    CHECK(oracle_sharpen_ex(big, W, H, PITCH, p.amount, p.gamma, p.osc_gain, p.osc_scale, ORACLE_READ_TRUNCATE, ref,
                            W, &S_ref, &m_ref) == 0,
          "oracle ex");
    sharp_layout L = {PITCH, 0, 1};
    CHECK(sharp_run_ex(ctx, big, &L, 1, 1, W, H, &p, SHARP_READ_TRUNCATE, out, &L) == SHARP_OK, "sharp_run_ex: %s",
          sharp_last_error(ctx));
    for (int r = 0; r < H; ++r) {
      compare(out + (size_t)r * PITCH, ref + (size_t)r * W, W, "sharp_run_ex row");
      for (int c = W; c < PITCH; ++c) CHECK(out[(size_t)r * PITCH + c] == 0xAB, "byte outside the ROI modified");
    }
    free(big);
    free(ref);
    free(out);
  }

  /* 5. the error contract */
  {
    uint8_t buf[64 * 64];
    CHECK(sharp_run(ctx, buf, 6, 64, &p, buf + 1) == SHARP_EINVAL, "w %% 4 != 0 must be EINVAL");
    CHECK(sharp_run(ctx, NULL, 64, 64, &p, buf) == SHARP_EINVAL, "NULL must be EINVAL");
    sharp_params bad = p;
    bad.gamma = -1.0f;
    CHECK(sharp_run(ctx, buf, 8, 8, &bad, buf + 100) == SHARP_EINVAL, "bad params must be EINVAL");
    CHECK(strcmp(sharp_strerror(SHARP_EINVAL), "invalid argument") == 0, "strerror");
  }

  sharp_destroy(ctx);

  /* 6. multi-device contexts (sharp_config.num_devices / device_ids / shard):
   *    a 2-way frame split, one image as 2 row bands, and device-resident
   *    bands.  On a one-GPU box both entries are device 0. */
  {
    int ndev = 0;
    CHECK(cudaGetDeviceCount(&ndev) == cudaSuccess && ndev >= 1, "cudaGetDeviceCount");
    int ids[2] = {0, 1 % ndev};
    sharp_config cfg;
    memset(&cfg, 0, sizeof(cfg));
    cfg.device = -1;
    cfg.num_devices = 2;
    cfg.device_ids = ids;
    cfg.shard = SHARP_SHARD_AUTO;
    sharp_ctx *m = NULL;
    CHECK(sharp_create(&m, &cfg) == SHARP_OK, "sharp_create (2 devices)");
    /* frames: 6 x 640x360 from host memory, 3 per device */
    {
      const int W = 640, H = 360, N = 6;
      const size_t fb = (size_t)W * H;
      uint8_t *imgs = malloc(N * fb), *ref = malloc(N * fb), *got = malloc(N * fb);
      synth_frames(imgs, N, W, H, 0, 0x5EED2015ull + 21, 0, 0);
      uint64_t sums[6], gsums[6];
      CHECK(oracle_sharpen_batch(imgs, N, W, H, p.amount, p.gamma, p.osc_gain, p.osc_scale, ref, sums, 0) == 0,
            "oracle batch");
      CHECK(sharp_run_batch(m, imgs, N, W, H, &p, got) == SHARP_OK, "multi-device batch: %s", sharp_last_error(m));
      compare(got, ref, N * fb, "frames split over 2 devices");
      CHECK(sharp_get_batch_sums(m, gsums, N) == SHARP_OK, "multi-device batch sums");
      for (int f = 0; f < N; ++f) CHECK(gsums[f] == sums[f], "S of frame %d (2 devices)", f);
      free(imgs);
      free(ref);
      free(got);
    }
    /* one 1920x1080 image: 2 row bands (AUTO for n == 1), host buffers */
    {
      const int W = 1920, H = 1080;
      const size_t n = (size_t)W * H;
      uint8_t *img = malloc(n), *ref = malloc(n), *got = malloc(n);
      synth_frames(img, 1, W, H, 0, 0x5EED2015ull + 22, 0, 0);
      uint64_t S_ref = 0;
      double m_ref = 0.0;
      CHECK(oracle_sharpen(img, W, H, p.amount, p.gamma, p.osc_gain, p.osc_scale, ref, &S_ref, &m_ref) == 0, "oracle");
      CHECK(sharp_run(m, img, W, H, &p, got) == SHARP_OK, "2 row bands: %s", sharp_last_error(m));
      compare(got, ref, n, "one image as 2 row bands");
      sharp_stats st;
      CHECK(sharp_get_stats(m, &st) == SHARP_OK && st.edge_sum == S_ref && st.edge_mean == m_ref, "2-band S / mean");
      /* the same image as device-resident bands (sharp_run_bands) */
      uint8_t *bands[2], *outs[2];
      int r0[2], r1[2];
      for (int g = 0; g < 2; ++g) {
        CHECK(sharp_band_rows(H, 2, g, &r0[g], &r1[g]) == SHARP_OK, "sharp_band_rows");
        const size_t bytes = (size_t)(r1[g] - r0[g]) * W;
        CHECK(cudaSetDevice(ids[g]) == cudaSuccess, "cudaSetDevice");
        CHECK(cudaMalloc((void **)&bands[g], bytes) == cudaSuccess && cudaMalloc((void **)&outs[g], bytes) == cudaSuccess,
              "band cudaMalloc");
        CHECK(cudaMemcpy(bands[g], img + (size_t)r0[g] * W, bytes, cudaMemcpyHostToDevice) == cudaSuccess, "band H2D");
      }
      CHECK(sharp_run_bands(m, (const uint8_t *const *)bands, W, H, &p, outs) == SHARP_OK, "sharp_run_bands: %s",
            sharp_last_error(m));
      memset(got, 0, n);
      for (int g = 0; g < 2; ++g) {
        CHECK(cudaSetDevice(ids[g]) == cudaSuccess, "cudaSetDevice");
        CHECK(cudaMemcpy(got + (size_t)r0[g] * W, outs[g], (size_t)(r1[g] - r0[g]) * W, cudaMemcpyDeviceToHost) ==
                  cudaSuccess,
              "band D2H");
        cudaFree(bands[g]);
        cudaFree(outs[g]);
      }
      compare(got, ref, n, "device-resident bands (sharp_run_bands)");
      free(img);
      free(ref);
      free(got);
    }
    sharp_destroy(m);
  }
  printf("c_abi_check ok (%s)\n", sharp_version());
  return 0;
}
