// Fused peer-memory exchange for row-band sharding of one image
// (DESIGN.md sec. 9): the two couplings between
// bands -- the 4 halo rows per side (L146 upscale, L158-L172 Sobel, L182
// window) and the global pEdge sum (L174) -- move by direct stores into the
// neighbours' / every rank's memory (NVLink peer mappings obtained with CUDA
// IPC), each published with an epoch flag, instead of NCCL send/recv and an
// NCCL all-reduce.  One single-CTA kernel per exchange; no host round trip.
//
// Window (symmetric layout, one per rank, allocated zeroed):
//   [0, 1024)   control (u64 words):
//                 [0, 64)  pEdge partial slots, two sets by epoch parity:
//                          slot[(e & 1) * 32 + g] = (e << 40) | S_g
//                 [64]     data_from_up    epoch of the rows in the upper halo
//                 [65]     data_from_down  epoch of the rows in the lower halo
//                 [66]     ready_up        the band above accepts this band's first rows of epoch e
//                 [67]     ready_down      the band below accepts this band's last rows of epoch e
//   [1024, ...) rows, pitch w: 4 halo rows (from the band above), the band's
//               own rows, 4 halo rows (from the band below)
// Handshake of epoch e (one single-CTA kernel per band): (1) tell both
// neighbours "my halos of epoch e-1 are consumed, push epoch e" (ready
// flags in THEIR windows), (2) wait for theirs, (3) push my edge rows into
// their halos, fence, set their data flags, (4) wait for my data flags.
// Every wait is on a flag a neighbour sets before it waits itself: no
// deadlock.  The partial slots are double-buffered by epoch parity: a rank
// can only write epoch e+1 after every rank's epoch-e partial reached it,
// and epoch e+2 only after this rank wrote e+1, i.e. after it read epoch e.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace sharp {
namespace {

constexpr int kSlots = 32;               // max ranks
constexpr int kDataUp = 2 * kSlots;      // rows from the band above are in my upper halo
constexpr int kDataDown = 2 * kSlots + 1;
constexpr int kReadyUp = 2 * kSlots + 2;   // the band above accepts my first rows
constexpr int kReadyDown = 2 * kSlots + 3; // the band below accepts my last rows
constexpr unsigned long long kSumMask = (1ull << 40) - 1;
static_assert((2 * kSlots + 4) * 8 <= kP2PCtlBytes, "control block");
static_assert(kDataUp == kCtlDataUp && kDataDown == kCtlDataDown && kReadyUp == kCtlReadyUp &&
                  kReadyDown == kCtlReadyDown && kSlots == kMaxRanks,
              "the fused band launch (kernels_tma.cu) uses the same window layout");

__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
// Spin until *p (acquire, system scope) satisfies `ok`; a peer that never
// arrives (a rank that died or skipped a call) traps after 10 s instead of
// hanging the device.
template <typename F>
__device__ __forceinline__ unsigned long long wait_flag(const unsigned long long *p, F ok) {
  const unsigned long long t0 = globaltimer_ns();
  unsigned long long v;
  while (!ok(v = ld_acquire_sys(p))) {
    __nanosleep(64);
    if (globaltimer_ns() - t0 > 10000000000ull) __trap();
  }
  return v;
}

// Halo exchange of epoch e for one band (see the handshake above).
// up / down: the neighbours' windows (peer mappings) or NULL; self: ours.
__global__ void p2p_halo_kernel(unsigned long long *self_ctl, const uint8_t *__restrict__ own, int w, int rows,
                                unsigned long long *up_ctl, uint8_t *up_halo, unsigned long long *down_ctl,
                                uint8_t *down_halo, unsigned long long epoch) {
  if (threadIdx.x == 0) {
    if (up_ctl) st_release_sys(up_ctl + kReadyDown, epoch);    // (1) the band above may fill my upper halo
    if (down_ctl) st_release_sys(down_ctl + kReadyUp, epoch);  //     the band below may fill my lower halo
    auto is_e = [epoch](unsigned long long v) { return v == epoch; };
    if (up_ctl) wait_flag(self_ctl + kReadyUp, is_e);  // (2)
    if (down_ctl) wait_flag(self_ctl + kReadyDown, is_e);
  }
  __syncthreads();
  const int n16 = (kP2PHalo * w) / 16;  // 16-byte words of 4 rows (w % 16 == 0)
  const uint4 *top = reinterpret_cast<const uint4 *>(own);
  const uint4 *bot = reinterpret_cast<const uint4 *>(own + (size_t)(rows - kP2PHalo) * w);
  for (int i = threadIdx.x; i < n16; i += blockDim.x) {  // (3)
    if (up_halo) reinterpret_cast<uint4 *>(up_halo)[i] = top[i];
    if (down_halo) reinterpret_cast<uint4 *>(down_halo)[i] = bot[i];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();  // the rows before the flags, for every observer
    if (up_ctl) st_release_sys(up_ctl + kDataDown, epoch);
    if (down_ctl) st_release_sys(down_ctl + kDataUp, epoch);
    auto is_e = [epoch](unsigned long long v) { return v == epoch; };
    if (up_ctl) wait_flag(self_ctl + kDataUp, is_e);  // (4)
    if (down_ctl) wait_flag(self_ctl + kDataDown, is_e);
  }
}

struct Peers {
  unsigned long long *slot[kSlots];  // &window_g.ctl.slot[rank] for every rank g
};

// The L174 reduction across bands: this band's partial goes to slot[rank] of
// every rank (itself included); then every slot of its own window must carry
// the epoch, and their sum is the image's S (identical on every rank).
__global__ void p2p_allreduce_kernel(Peers peers, int G, const unsigned long long *partial,
                                     const unsigned long long *my_slots, unsigned long long epoch,
                                     unsigned long long *total) {
  __shared__ unsigned long long part[kSlots];
  const int t = threadIdx.x;
  if (t < G) {
    st_release_sys(peers.slot[t], (epoch << 40) | (*partial & kSumMask));
    const unsigned long long v =
        wait_flag(my_slots + t, [epoch](unsigned long long x) { return (x >> 40) == (epoch & 0xffffffull); });
    part[t] = v & kSumMask;
  }
  __syncthreads();
  if (t == 0) {
    unsigned long long s = 0;
    for (int g = 0; g < G; ++g) s += part[g];
    *total = s;
  }
}

}  // namespace

size_t p2p_window_bytes(int w, int rows_own) { return kP2PCtlBytes + (size_t)(rows_own + 2 * kP2PHalo) * w; }

cudaError_t launch_p2p_halo(uint8_t *self, int w, int rows_own, uint8_t *up, int up_rows_own, uint8_t *down,
                            unsigned long long epoch, cudaStream_t st) {
  auto ctl = [](uint8_t *win) { return reinterpret_cast<unsigned long long *>(win); };
  auto rows = [](uint8_t *win) { return win + kP2PCtlBytes; };
  const uint8_t *own = rows(self) + (size_t)kP2PHalo * w;
  uint8_t *up_halo = up ? rows(up) + (size_t)(kP2PHalo + up_rows_own) * w : nullptr;  // its lower halo
  uint8_t *down_halo = down ? rows(down) : nullptr;                                   // its upper halo
  p2p_halo_kernel<<<1, 512, 0, st>>>(ctl(self), own, w, rows_own, up ? ctl(up) : nullptr, up_halo,
                                     down ? ctl(down) : nullptr, down_halo, epoch);
  return cudaGetLastError();
}

cudaError_t launch_p2p_allreduce(uint8_t *const *windows, int G, int rank, const unsigned long long *partial,
                                 unsigned long long epoch, unsigned long long *total, cudaStream_t st) {
  if (G < 1 || G > kSlots || rank < 0 || rank >= G) return cudaErrorInvalidValue;
  const int set = (int)(epoch & 1) * kSlots;
  Peers p{};
  for (int g = 0; g < G; ++g) p.slot[g] = reinterpret_cast<unsigned long long *>(windows[g]) + set + rank;
  p2p_allreduce_kernel<<<1, 32, 0, st>>>(p, G, partial,
                                          reinterpret_cast<const unsigned long long *>(windows[rank]) + set,
                                          epoch & 0xffffffull, total);
  return cudaGetLastError();
}

// Forces the (lazy) module load of this file's kernels; see kernels.h.
cudaError_t preload_p2p() {
  cudaFuncAttributes a;
  cudaError_t e;
  if ((e = cudaFuncGetAttributes(&a, p2p_halo_kernel)) != cudaSuccess) return e;
  if ((e = cudaFuncGetAttributes(&a, p2p_allreduce_kernel)) != cudaSuccess) return e;
  return cudaSuccess;
}

}  // namespace sharp
