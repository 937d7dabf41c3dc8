// prep.cu — B1: the lookback-2 pair table (§IV-A), built once per DFA
// at load time (preparation is excluded from timing).
//
// For every pair of byte classes (a, b): run all real states q over (a, b),
// count how often each end state appears, and keep the distinct end states
// ranked by (-multiplicity, transformed id) — QS_c for any chunk whose two
// preceding symbols fall in (a, b).  A chunk's prediction is then one gather
// instead of 2n transitions.
#include <algorithm>

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

// Full lookback-2 images with multiplicities (for lookbacks longer than 2, reading R25):
// per class pair, the distinct end states of all real states over (a, b) and how many
// states reach each, when there are at most kImgFull of them (img_n = 0xFF: wider).
__global__ void __launch_bounds__(kPB) k_build_img2(const uint32_t* __restrict__ ttc, uint32_t n, uint32_t nt,
                                                   uint32_t C, uint32_t* __restrict__ scratch,
                                                   uint32_t* __restrict__ img_s, uint32_t* __restrict__ img_m,
                                                   uint8_t* __restrict__ img_n) {
  uint32_t* mult = scratch + (uint64_t)blockIdx.x * nt;
  __shared__ uint32_t cnt;
  const uint32_t npairs = C * C;
  for (uint32_t pr = blockIdx.x; pr < npairs; pr += gridDim.x) {
    const uint32_t a = pr / C, b = pr % C;
    for (uint32_t s = threadIdx.x; s < nt; s += kPB) mult[s] = 0;
    if (threadIdx.x == 0) cnt = 0;
    __syncthreads();
    for (uint32_t q = threadIdx.x; q < n; q += kPB) atomicAdd(mult + ttc[(uint64_t)ttc[(uint64_t)q * C + a] * C + b], 1u);
    __syncthreads();
    for (uint32_t s = threadIdx.x; s < nt; s += kPB)
      if (mult[s]) {
        const uint32_t i = atomicAdd(&cnt, 1u);
        if (i < kImgFull) {
          img_s[(uint64_t)pr * kImgFull + i] = s;
          img_m[(uint64_t)pr * kImgFull + i] = mult[s];
        }
      }
    __syncthreads();
    if (threadIdx.x == 0) img_n[pr] = cnt <= kImgFull ? (uint8_t)cnt : (uint8_t)0xFF;
    __syncthreads();
  }
}

// Lookback-L prediction per chunk (P:300 with L > 2, reading R25), one warp per chunk
// c >= 1: the window w = in[cB - L, cB); the multiset image of all real states over w is
// the pair image of (w_0, w_1) with multiplicities walked over w_2 .. w_{L-1} (composition
// of transitions), merged by end state and ranked by (-multiplicity, id); the top kQsMax
// go to qsc[c].  A pair image wider than kImgFull keeps the lookback-2 ranking of the last
// two symbols (it contains the true start as well).
__global__ void __launch_bounds__(256) k_qs_long(DevImage img, const uint32_t* __restrict__ ttc,
                                                 const uint8_t* __restrict__ in, uint32_t B, uint64_t N, uint32_t L,
                                                 const uint32_t* __restrict__ img_s, const uint32_t* __restrict__ img_m,
                                                 const uint8_t* __restrict__ img_n, uint32_t* __restrict__ qsc,
                                                 uint8_t* __restrict__ qsc_len) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t w0 = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) / 32, nw = (uint64_t)gridDim.x * blockDim.x / 32;
  for (uint64_t c = w0; c < N; c += nw) {
    if (c == 0) continue;  // chunk 0 starts at q0
    const uint8_t* w = in + c * (uint64_t)B - L;
    const uint32_t pr = (uint32_t)__ldg(img.cls + w[0]) * img.C + __ldg(img.cls + w[1]);
    const uint32_t n2 = __ldg(img_n + pr);
    if (n2 == 0xFF) {  // wide: the lookback-2 ranking of the last two symbols
      const uint32_t p2 = (uint32_t)__ldg(img.cls + w[L - 2]) * img.C + __ldg(img.cls + w[L - 1]);
      if (lane < kQsMax) qsc[c * kQsMax + lane] = __ldg(img.qs2 + (uint64_t)p2 * kQsMax + lane);
      if (lane == 0) qsc_len[c] = __ldg(img.qs2_len + p2);
      continue;
    }
    // two entries per lane: e = lane, lane + 32
    uint32_t s[2], m[2];
#pragma unroll
    for (int h = 0; h < 2; h++) {
      const uint32_t e = lane + 32 * h;
      s[h] = e < n2 ? __ldg(img_s + (uint64_t)pr * kImgFull + e) : 0u;
      m[h] = e < n2 ? __ldg(img_m + (uint64_t)pr * kImgFull + e) : 0u;
      if (m[h])
        for (uint32_t i = 2; i < L; i++) s[h] = __ldg(ttc + (uint64_t)s[h] * img.C + __ldg(img.cls + w[i]));
    }
    // merge equal end states: the first entry of a group leads and sums the multiplicities
    // (n2 is warp-uniform: the loops run over the pair image's entries only)
    uint32_t tot[2] = {0, 0};
    bool lead[2] = {m[0] != 0, m[1] != 0};
    for (uint32_t k = 0; k < n2; k++) {
      const uint32_t sk = __shfl_sync(0xffffffffu, s[k >> 5], k & 31);
      const uint32_t mk = __shfl_sync(0xffffffffu, m[k >> 5], k & 31);
#pragma unroll
      for (int h = 0; h < 2; h++)
        if (mk && m[h] && sk == s[h]) {
          tot[h] += mk;
          if (k < lane + 32 * h) lead[h] = false;
        }
    }
    // rank the leaders by (-multiplicity, id)
    uint32_t rank[2] = {0, 0}, nlead = 0;
    for (uint32_t k = 0; k < n2; k++) {
      const uint32_t sk = __shfl_sync(0xffffffffu, s[k >> 5], k & 31);
      const uint32_t tk = __shfl_sync(0xffffffffu, tot[k >> 5], k & 31);
      const bool lk = __shfl_sync(0xffffffffu, (uint32_t)lead[k >> 5], k & 31) != 0;
      nlead += lk;
#pragma unroll
      for (int h = 0; h < 2; h++)
        if (lk && lead[h] && (tk > tot[h] || (tk == tot[h] && sk < s[h]))) rank[h]++;
    }
#pragma unroll
    for (int h = 0; h < 2; h++)
      if (lead[h] && rank[h] < kQsMax) qsc[c * kQsMax + rank[h]] = s[h];
    if (lane == 0) qsc_len[c] = (uint8_t)min(nlead, kQsMax);
  }
}

}  // namespace

cudaError_t launch_build_img2_raw(const uint32_t* d_ttc, uint32_t n, uint32_t C, uint32_t* scratch, uint32_t grid,
                                  uint32_t* img_s, uint32_t* img_m, uint8_t* img_n, cudaStream_t st) {
  k_build_img2<<<grid, kPB, 0, st>>>(d_ttc, n, n + 1, C, scratch, img_s, img_m, img_n);
  return cudaGetLastError();
}

cudaError_t launch_qs_long(const DevImage& img, const uint32_t* d_ttc, const uint8_t* in, uint32_t B, uint64_t N,
                           uint32_t L, const uint32_t* img_s, const uint32_t* img_m, const uint8_t* img_n,
                           uint32_t* qsc, uint8_t* qsc_len, int sms, cudaStream_t st) {
  if (N < 2) return cudaSuccess;
  const uint64_t grid = std::min<uint64_t>((N * 32 + 255) / 256, (uint64_t)sms * 16);
  k_qs_long<<<(unsigned)grid, 256, 0, st>>>(img, d_ttc, in, B, N, L, img_s, img_m, img_n, qsc, qsc_len);
  return cudaGetLastError();
}

cudaError_t launch_build_qs2_raw(const uint32_t* d_ttc, uint32_t n, uint32_t C, uint32_t* scratch,
                                 uint32_t grid, uint32_t* qs2, uint8_t* qs2_len, uint32_t* qs2_img,
                                 cudaStream_t st) {
  k_build_qs2<<<grid, kPB, 0, st>>>(d_ttc, n, n + 1, C, scratch, qs2, qs2_len, qs2_img);
  return cudaGetLastError();
}

}  // namespace gspec
