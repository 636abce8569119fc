// Minimal compute-sanitizer racecheck repro of the step kernel's stage
// hand-off (tools/README.md): a producer thread writes a shared word and
// arrives on a "full" mbarrier; a consumer WARP waits on it, every lane reads
// the word, and the warp frees the slot on an "empty" mbarrier that the
// producer waits on before the next write.  Both variants are correct under
// the PTX memory model; they differ only in who arrives on "empty":
//   mode 0: lane 0 after __syncwarp() (the step kernel's pattern; empty count 1)
//   mode 1: every lane (empty count 32)
// racecheck reports WAR hazards for mode 0 only: it does not carry the other
// lanes' reads through bar.warp.sync into lane 0's release.
#include <cstdint>
#include <cstdio>
#include <cstdlib>
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(n));
}
__device__ __forceinline__ void arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void wait(uint32_t bar, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                   bar),
               "r"(par)
               : "memory");
}
__global__ void k(int *out, int rounds, int mode) {
  __shared__ __align__(8) unsigned long long bars[2];
  __shared__ int slot;
  const uint32_t full = (uint32_t)__cvta_generic_to_shared(&bars[0]), empty = (uint32_t)__cvta_generic_to_shared(&bars[1]);
  if (threadIdx.x == 0) {
    mbar_init(full, 1);
    mbar_init(empty, mode ? 32 : 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  int acc = 0;
  for (int i = 0; i < rounds; ++i) {
    if (threadIdx.x == 32) {  // producer thread (warp 1)
      if (i) wait(empty, (i - 1) & 1);
      slot = i + 1;
      arrive(full);
    }
    if (threadIdx.x < 32) {  // consumer warp (warp 0)
      wait(full, i & 1);
      acc += slot;
      if (mode) {
        arrive(empty);
      } else {
        __syncwarp();
        if (threadIdx.x == 0) arrive(empty);
      }
    }
  }
  if (threadIdx.x < 32) atomicAdd(out, acc);
}
int main(int argc, char **argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  int *d;
  cudaMalloc(&d, 4);
  cudaMemset(d, 0, 4);
  k<<<1, 64>>>(d, 8, mode);
  int h = 0;
  cudaMemcpy(&h, d, 4, cudaMemcpyDeviceToHost);
  printf("mode %d: sum %d (expected %d) %s\n", mode, h, 32 * 36, cudaGetErrorString(cudaGetLastError()));
  return h == 32 * 36 ? 0 : 1;
}
