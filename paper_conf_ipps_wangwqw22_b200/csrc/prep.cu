// prep.cu — B1: the lookback-2 pair table (§IV-A), built once per DFA
// at load time (preparation is excluded from timing).
//
// For every pair of byte classes (a, b): run all real states q over (a, b),
// count how often each end state appears, and keep the distinct end states
// ranked by (-multiplicity, transformed id) — QS_c for any chunk whose two
// preceding symbols fall in (a, b).  A chunk's prediction is then one gather
// instead of 2n transitions.
#include "internal.h"

namespace gspec {
namespace {

constexpr int kPB = 256;

__global__ void __launch_bounds__(kPB) k_build_qs2(const uint32_t* __restrict__ ttc, uint32_t n, uint32_t nt,
                                                  uint32_t C, uint32_t* __restrict__ scratch,
                                                  uint32_t* __restrict__ qs2, uint8_t* __restrict__ qs2_len,
                                                  uint32_t* __restrict__ qs2_img) {
  uint32_t* mult = scratch + (uint64_t)blockIdx.x * nt;
  __shared__ unsigned long long red[kPB / 32];
  __shared__ uint32_t sh_img;
  const uint32_t npairs = C * C;
  for (uint32_t pr = blockIdx.x; pr < npairs; pr += gridDim.x) {
    const uint32_t a = pr / C, b = pr % C;
    for (uint32_t s = threadIdx.x; s < nt; s += kPB) mult[s] = 0;
    __syncthreads();
    for (uint32_t q = threadIdx.x; q < n; q += kPB) {
      const uint32_t s = ttc[(uint64_t)ttc[(uint64_t)q * C + a] * C + b];
      atomicAdd(mult + s, 1u);
    }
    __syncthreads();
    uint32_t nz = 0;
    for (uint32_t s = threadIdx.x; s < nt; s += kPB) nz += mult[s] != 0;
    for (int o = 16; o > 0; o >>= 1) nz += __shfl_down_sync(0xffffffffu, nz, o);
    if (threadIdx.x == 0) sh_img = 0;
    __syncthreads();
    if ((threadIdx.x & 31) == 0) atomicAdd(&sh_img, nz);
    __syncthreads();
    const uint32_t img = sh_img;
    const uint32_t K = img < kQsMax ? img : kQsMax;
    for (uint32_t r = 0; r < K; r++) {
      // key = (mult << 32) | (~id): max key = largest multiplicity, then lowest id
      unsigned long long best = 0;
      for (uint32_t s = threadIdx.x; s < nt; s += kPB) {
        const uint32_t m = mult[s];
        if (m) {
          const unsigned long long key = ((unsigned long long)m << 32) | (0xFFFFFFFFu - s);
          best = key > best ? key : best;
        }
      }
      for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long y = __shfl_down_sync(0xffffffffu, best, o);
        best = y > best ? y : best;
      }
      if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = best;
      __syncthreads();
      if (threadIdx.x == 0) {
        unsigned long long bb = 0;
        for (int w = 0; w < kPB / 32; w++) bb = red[w] > bb ? red[w] : bb;
        const uint32_t s = 0xFFFFFFFFu - (uint32_t)(bb & 0xFFFFFFFFu);
        qs2[(uint64_t)pr * kQsMax + r] = s;
        mult[s] = 0;
      }
      __syncthreads();
    }
    if (threadIdx.x == 0) {
      for (uint32_t r = K; r < kQsMax; r++) qs2[(uint64_t)pr * kQsMax + r] = n;  // padding: poison
      qs2_len[pr] = (uint8_t)K;
      qs2_img[pr] = img;
    }
    __syncthreads();
  }
}

}  // namespace

cudaError_t launch_build_qs2_raw(const uint32_t* d_ttc, uint32_t n, uint32_t C, uint32_t* scratch,
                                 uint32_t grid, uint32_t* qs2, uint8_t* qs2_len, uint32_t* qs2_img,
                                 cudaStream_t st) {
  k_build_qs2<<<grid, kPB, 0, st>>>(d_ttc, n, n + 1, C, scratch, qs2, qs2_len, qs2_img);
  return cudaGetLastError();
}

}  // namespace gspec
