// General layouts (reading R1'): the
// fused kernels take dense [n][H][W] frames with W, H multiples of 4.  A
// strided / pitched / interleaved-channel source, or a size that is not a
// multiple of 4, is gathered into that form first -- unit u = f * C + c is
// channel c of frame f, extended to W4 x H4 (the next multiples of 4) by
// replicating its last column and last row -- and the top-left w x h of each
// dense result is scattered back into the caller's layout.  Plain byte
// copies; the benchmarked dense path never runs them.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace sharp {
namespace {

// A block per (unit, row) pair (grid-stride over rows), threads across the
// row: no 64-bit index divisions per byte.

// Dense padded row r of unit u <- source row min(r, h-1), columns clamped to
// w-1 (replicate, R1'); one 32-bit store per 4 bytes.
__global__ void gather_kernel(const uint8_t *__restrict__ src, size_t fs, size_t pitch, int es, int C, int w, int h,
                              int W4, int H4, int P, int units, uint8_t *__restrict__ dst) {
  const int q4 = W4 >> 2;
  for (unsigned ur = blockIdx.x; ur < (unsigned)units * (unsigned)H4; ur += gridDim.x) {
    const unsigned u = ur / (unsigned)H4, r = ur - u * (unsigned)H4;
    const uint8_t *row = src + (size_t)(u / C) * fs + (size_t)(u % C) + (size_t)min((int)r, h - 1) * pitch;
    uint32_t *drow = reinterpret_cast<uint32_t *>(dst + (size_t)ur * P);
    for (int q = threadIdx.x; q < q4; q += blockDim.x) {
      uint32_t v = 0;
      if (es == 1 && 4 * q + 3 < w) {
        // 4 contiguous source bytes: the aligned word(s) holding them and a
        // funnel shift (an aligned word with a valid byte never crosses a page)
        const uintptr_t a = (uintptr_t)(row + 4 * q);
        const uint32_t *al = reinterpret_cast<const uint32_t *>(a & ~(uintptr_t)3);
        const uint32_t sh = (uint32_t)(a & 3) * 8;
        v = sh ? __funnelshift_r(al[0], al[1], sh) : al[0];
      } else {
#pragma unroll
        for (int k = 0; k < 4; ++k) v |= (uint32_t)row[(size_t)min(4 * q + k, w - 1) * es] << (8 * k);
      }
      drow[q] = v;
    }
  }
}

// Single-channel rows (elem_stride 1): per destination row, 16-byte stores
// where the destination is aligned (the row interior), bytes at the ends.
__global__ void scatter_rows_kernel(const uint8_t *__restrict__ src, int P, int H4, int units, int w, int h,
                                    uint8_t *__restrict__ dst, size_t fs, size_t pitch) {
  for (unsigned ur = blockIdx.x; ur < (unsigned)units * (unsigned)h; ur += gridDim.x) {
    const unsigned u = ur / (unsigned)h, r = ur - u * (unsigned)h;
    uint8_t *drow = dst + (size_t)u * fs + (size_t)r * pitch;
    const uint8_t *srow = src + ((size_t)u * H4 + r) * P;
    const int lead = min(w, (int)((16 - ((uintptr_t)drow & 15)) & 15));  // bytes before the first aligned one
    const int nvec = (w - lead) / 16;
    for (int c = threadIdx.x; c < lead; c += blockDim.x) drow[c] = srow[c];
    for (int k = threadIdx.x; k < nvec; k += blockDim.x) {
      const int c0 = lead + 16 * k;
      uint4 v;
      uint8_t *b = reinterpret_cast<uint8_t *>(&v);
#pragma unroll
      for (int j = 0; j < 16; ++j) b[j] = srow[c0 + j];
      *reinterpret_cast<uint4 *>(drow + c0) = v;
    }
    for (int c = lead + 16 * nvec + threadIdx.x; c < w; c += blockDim.x) drow[c] = srow[c];
  }
}

// Any layout (interleaved channels): a byte per thread.
__global__ void scatter_kernel(const uint8_t *__restrict__ src, int P, int H4, int units, int w, int h,
                               uint8_t *__restrict__ dst, size_t fs, size_t pitch, int es, int C) {
  for (unsigned ur = blockIdx.x; ur < (unsigned)units * (unsigned)h; ur += gridDim.x) {
    const unsigned u = ur / (unsigned)h, r = ur - u * (unsigned)h;
    uint8_t *drow = dst + (size_t)(u / C) * fs + (size_t)(u % C) + (size_t)r * pitch;
    const uint8_t *srow = src + ((size_t)u * H4 + r) * P;
    for (int c = threadIdx.x; c < w; c += blockDim.x) drow[(size_t)c * es] = srow[c];
  }
}

unsigned rows_grid(size_t rows) { return (unsigned)(rows < 148 * 16 ? (rows ? rows : 1) : 148 * 16); }

}  // namespace

cudaError_t launch_gather(const uint8_t *src, size_t frame_stride, size_t pitch, int elem_stride, int C, int w,
                          int h, int W4, int H4, int P, int units, uint8_t *dst, cudaStream_t st) {
  gather_kernel<<<rows_grid((size_t)units * H4), 128, 0, st>>>(src, frame_stride, pitch, elem_stride, C, w, h, W4, H4,
                                                                P, units, dst);
  return cudaGetLastError();
}

cudaError_t launch_scatter(const uint8_t *src, int P, int H4, int units, int w, int h, uint8_t *dst,
                           size_t frame_stride, size_t pitch, int elem_stride, int C, cudaStream_t st) {
  if (elem_stride == 1 && C == 1)
    scatter_rows_kernel<<<rows_grid((size_t)units * h), 128, 0, st>>>(src, P, H4, units, w, h, dst, frame_stride,
                                                                       pitch);
  else
    scatter_kernel<<<rows_grid((size_t)units * h), 128, 0, st>>>(src, P, H4, units, w, h, dst, frame_stride, pitch,
                                                                  elem_stride, C);
  return cudaGetLastError();
}

cudaError_t preload_layout() {
  cudaFuncAttributes a;
  cudaError_t e;
  if ((e = cudaFuncGetAttributes(&a, gather_kernel)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, scatter_rows_kernel)) != cudaSuccess) return e;
  return cudaFuncGetAttributes(&a, scatter_kernel);
}

}  // namespace sharp
