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

// One thread per 4 dense output bytes (one 32-bit store), grid-stride.
__global__ void gather_kernel(const uint8_t *__restrict__ src, size_t fs, size_t pitch, int es, int C, int w, int h,
                              int W4, int H4, int units, uint8_t *__restrict__ dst) {
  const int q4 = W4 >> 2;
  const size_t total = (size_t)units * H4 * q4;
  for (size_t t = blockIdx.x * (size_t)blockDim.x + threadIdx.x; t < total; t += (size_t)gridDim.x * blockDim.x) {
    const int q = (int)(t % q4);
    const size_t ur = t / q4;
    const int r = (int)(ur % H4), u = (int)(ur / H4);
    const uint8_t *row = src + (size_t)(u / C) * fs + (size_t)(u % C) + (size_t)min(r, h - 1) * pitch;
    uint32_t v = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) v |= (uint32_t)row[(size_t)min(4 * q + k, w - 1) * es] << (8 * k);
    reinterpret_cast<uint32_t *>(dst)[t] = v;
  }
}

// One thread per output byte of the w x h crop, grid-stride.
__global__ void scatter_kernel(const uint8_t *__restrict__ src, int W4, int H4, int units, int w, int h,
                               uint8_t *__restrict__ dst, size_t fs, size_t pitch, int es, int C) {
  const size_t total = (size_t)units * h * w;
  for (size_t t = blockIdx.x * (size_t)blockDim.x + threadIdx.x; t < total; t += (size_t)gridDim.x * blockDim.x) {
    const int c = (int)(t % w);
    const size_t ur = t / w;
    const int r = (int)(ur % h), u = (int)(ur / h);
    dst[(size_t)(u / C) * fs + (size_t)(u % C) + (size_t)r * pitch + (size_t)c * es] =
        src[((size_t)u * H4 + r) * W4 + c];
  }
}

unsigned grid_for(size_t work) {
  const size_t b = (work + 255) / 256;
  return (unsigned)(b < 148 * 32 ? (b ? b : 1) : 148 * 32);
}

}  // namespace

cudaError_t launch_gather(const uint8_t *src, size_t frame_stride, size_t pitch, int elem_stride, int C, int w,
                          int h, int W4, int H4, int units, uint8_t *dst, cudaStream_t st) {
  gather_kernel<<<grid_for((size_t)units * H4 * (W4 / 4)), 256, 0, st>>>(src, frame_stride, pitch, elem_stride, C, w,
                                                                         h, W4, H4, units, dst);
  return cudaGetLastError();
}

cudaError_t launch_scatter(const uint8_t *src, int W4, int H4, int units, int w, int h, uint8_t *dst,
                           size_t frame_stride, size_t pitch, int elem_stride, int C, cudaStream_t st) {
  scatter_kernel<<<grid_for((size_t)units * h * w), 256, 0, st>>>(src, W4, H4, units, w, h, dst, frame_stride, pitch,
                                                                   elem_stride, C);
  return cudaGetLastError();
}

cudaError_t preload_layout() {
  cudaFuncAttributes a;
  cudaError_t e;
  if ((e = cudaFuncGetAttributes(&a, gather_kernel)) != cudaSuccess) return e;
  return cudaFuncGetAttributes(&a, scatter_kernel);
}

}  // namespace sharp
