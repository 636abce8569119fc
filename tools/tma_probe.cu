// Minimal TMA probe: which tensor-map / box configurations load correctly.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdint.h>
#include <vector>
#include <stdlib.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void probe(const __grid_constant__ CUtensorMap m, int c, int r, uint8_t* out, int nbytes) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&bar)), "r"(nbytes) : "memory");
    if (MODE == 3)
      asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                   :: "r"(su(sm)), "l"(&m), "r"(c), "r"(r), "r"(0), "r"(su(&bar)) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                   :: "r"(su(sm)), "l"(&m), "r"(c), "r"(r), "r"(su(&bar)) : "memory");
  }
  asm volatile("{ .reg .pred p; W_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0; @!p bra W_%=; }" :: "r"(su(&bar)) : "memory");
  for (int i = threadIdx.x; i < nbytes; i += blockDim.x) out[i] = sm[i];
}

int main(int argc, char** argv) {
  cudaDriverEntryPointQueryResult q; void* p = nullptr;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)p;
  struct Case { int W, H, bw, bh, dims, c, r; };
  Case cases[] = {{1024, 64, 256, 40, 2, 0, 0}, {1024, 64, 256, 40, 2, -8, -4}, {16, 16, 256, 40, 2, 0, 0},
                  {16, 16, 256, 40, 2, -8, -4}, {1024, 64, 256, 40, 3, -8, -4}, {16, 16, 256, 40, 3, -8, -4},
                  {16, 16, 16, 8, 2, 0, 0}, {1024, 64, 128, 40, 2, 0, 0}};
  if (argc > 1) {  // one custom case: W H bw bh dims c r
    Case c1{atoi(argv[1]), atoi(argv[2]), atoi(argv[3]), atoi(argv[4]), atoi(argv[5]), atoi(argv[6]), atoi(argv[7])};
    cases[0] = c1;
  }
  int ncase = argc > 1 ? 1 : (int)(sizeof(cases) / sizeof(cases[0]));
  for (int ci = 0; ci < ncase; ++ci) {
    auto& cs = cases[ci];
    std::vector<uint8_t> h(cs.W * cs.H);
    for (int i = 0; i < cs.W * cs.H; ++i) h[i] = (uint8_t)(i * 7 + 3);
    uint8_t *d, *o; cudaMalloc(&d, h.size()); cudaMalloc(&o, 256 * 256);
    cudaMemcpy(d, h.data(), h.size(), cudaMemcpyHostToDevice);
    CUtensorMap m;
    cuuint64_t dims[3] = {(cuuint64_t)cs.W, (cuuint64_t)cs.H, 1};
    cuuint64_t str[2] = {(cuuint64_t)cs.W, (cuuint64_t)cs.W * cs.H};
    cuuint32_t box[3] = {(cuuint32_t)cs.bw, (cuuint32_t)cs.bh, 1};
    cuuint32_t es[3] = {1, 1, 1};
    CUresult er = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, cs.dims, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    int nb = cs.bw * cs.bh;
    cudaFuncSetAttribute(probe<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
    cudaFuncSetAttribute(probe<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
    if (cs.dims == 3) probe<3><<<1, 128, nb>>>(m, cs.c, cs.r, o, nb); else probe<2><<<1, 128, nb>>>(m, cs.c, cs.r, o, nb);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<uint8_t> got(nb); cudaMemcpy(got.data(), o, nb, cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int y = 0; y < cs.bh; ++y) for (int x = 0; x < cs.bw; ++x) {
      int gx = cs.c + x, gy = cs.r + y;
      uint8_t ex = (gx >= 0 && gx < cs.W && gy >= 0 && gy < cs.H) ? h[gy * cs.W + gx] : 0;
      bad += got[y * cs.bw + x] != ex;
    }
    printf("W=%d H=%d box=%dx%d dims=%d at (%d,%d): encode=%d launch=%s bad=%d\n", cs.W, cs.H, cs.bw, cs.bh, cs.dims,
           cs.c, cs.r, (int)er, cudaGetErrorString(e), bad);
    if (e != cudaSuccess) return 1;
    cudaFree(d); cudaFree(o);
  }
  return 0;
}
