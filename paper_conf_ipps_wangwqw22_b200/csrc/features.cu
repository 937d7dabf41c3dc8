// features.cu — B6: selector features (Table II; reading R19).
//  * spec-1 / spec-k accuracy of the lookback predictor against the true chunk
//    starts of an exact run on the profile sample, per 8 segments (input
//    sensitivity = max - min of per-segment spec-1 accuracy);
//  * uniq10: #unique states after 10 transitions from all states, averaged
//    over 64 evenly spaced positions (a lightweight convergence profile);
//  * convergence lengths of the lookback image (reading R29) -> chunk size.
#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

// counts: [0..8) seg hits, [8..16) seg totals, [16] hit1, [17] hitk
__global__ void k_feat_acc(DevImage img, const uint8_t* __restrict__ in, uint32_t B, uint64_t N,
                           const uint32_t* __restrict__ x, uint32_t k, uint32_t qs_cap,
                           unsigned long long* __restrict__ counts) {
  for (uint64_t c = 1 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < N; c += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t pair = qs_pair(img, in, c, B);
    const uint32_t ql = min((uint32_t)img.qs2_len[pair], qs_cap);
    const uint32_t truth = x[c];
    const uint32_t* qs = img.qs2 + (uint64_t)pair * kQsMax;
    const bool h1 = ql > 0 && qs[0] == truth;
    bool hk = false;
    for (uint32_t j = 0; j < ql && j < k; j++) hk |= qs[j] == truth;
    const uint64_t sg = N > 1 ? ((c - 1) * 8) / (N - 1) : 0;
    if (h1) { atomicAdd(counts + sg, 1ull); atomicAdd(counts + 16, 1ull); }
    if (hk) atomicAdd(counts + 17, 1ull);
    atomicAdd(counts + 8 + sg, 1ull);
  }
}

// one block per position j < 64; seen: 64 bitmaps of nt bits (zeroed by caller)
__global__ void k_feat_uniq(DevImage img, const uint32_t* __restrict__ ttc, const uint8_t* __restrict__ in,
                            uint64_t len, uint32_t* __restrict__ seen, unsigned long long* __restrict__ uniq) {
  const uint32_t nt = img.n + 1, words = (nt + 31) / 32;
  const uint64_t p = (uint64_t)blockIdx.x * (len - 10) / 64;
  uint32_t* bm = seen + (uint64_t)blockIdx.x * words;
  __shared__ uint8_t cl[10];
  if (threadIdx.x < 10) cl[threadIdx.x] = img.cls[in[p + threadIdx.x]];
  __syncthreads();
  uint32_t u = 0;
  for (uint32_t q = threadIdx.x; q < img.n; q += blockDim.x) {
    uint32_t t = q;
    for (int i = 0; i < 10; i++) t = ttc[(uint64_t)t * img.C + cl[i]];
    const uint32_t old = atomicOr(bm + t / 32, 1u << (t % 32));
    u += (old & (1u << (t % 32))) == 0;
  }
  for (int o = 16; o > 0; o >>= 1) u += __shfl_down_sync(0xffffffffu, u, o);
  if ((threadIdx.x & 31) == 0 && u) atomicAdd(uniq, (unsigned long long)u);
}

// Convergence length of the lookback image (reading R29): one warp per window w (start
// p = 4096 j, j = 32 (w / 28) + 1 + w % 28, so a window stays inside one 128 KiB profile
// portion); lane i walks the i-th ranked state of the window's lookback-2 image (lanes past
// the image repeat state 0), and after every 64 bytes the warp votes whether every path is
// in one state.  dout[w] = bytes to that point, 0 for a one-state image, ~0 past wmax.
__global__ void k_feat_conv(DevImage img, const uint32_t* __restrict__ ttc, const uint8_t* __restrict__ in,
                            uint32_t nwin, uint32_t wmax, uint32_t* __restrict__ dout) {
  const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (w >= nwin) return;
  const uint64_t p = ((uint64_t)(w / 28) * 32 + 1 + w % 28) * 4096;
  const uint32_t pair = (uint32_t)img.cls[in[p - 2]] * img.C + img.cls[in[p - 1]];
  const uint32_t ql = min((uint32_t)img.qs2_len[pair], (uint32_t)kQsMax);
  uint32_t d = 0;
  if (ql > 1) {
    uint32_t t = img.qs2[(uint64_t)pair * kQsMax + (lane < ql ? lane : 0)];
    d = 0xFFFFFFFFu;
    for (uint32_t i = 0; i < wmax; i += 64) {
      for (uint32_t k = 0; k < 64; k++) t = ttc[(uint64_t)t * img.C + img.cls[in[p + i + k]]];
      if (__all_sync(0xffffffffu, t == __shfl_sync(0xffffffffu, t, 0))) {
        d = i + 64;
        break;
      }
    }
  }
  if (lane == 0) dout[w] = d;
}

}  // namespace

cudaError_t launch_feat_conv(const DevImage& img, const uint32_t* d_ttc, const uint8_t* in, uint32_t nwin,
                             uint32_t wmax, uint32_t* d_out, cudaStream_t st) {
  if (nwin == 0) return cudaSuccess;
  k_feat_conv<<<(nwin + 3) / 4, 128, 0, st>>>(img, d_ttc, in, nwin, wmax, d_out);
  return cudaGetLastError();
}

cudaError_t launch_features_raw(const DevImage& img, const uint32_t* d_ttc, const uint8_t* in, uint64_t len,
                                uint32_t B, uint64_t N, const uint32_t* d_x, uint32_t k, uint32_t qs_cap,
                                unsigned long long* d_counts, uint32_t* d_seen, unsigned long long* d_uniq,
                                cudaStream_t st) {
  if (N > 1) {
    uint64_t grid = (N + 255) / 256;
    if (grid > 148 * 8) grid = 148 * 8;
    k_feat_acc<<<(unsigned)grid, 256, 0, st>>>(img, in, B, N, d_x, k, qs_cap, d_counts);
  }
  if (len >= 10) k_feat_uniq<<<64, 256, 0, st>>>(img, d_ttc, in, len, d_seen, d_uniq);
  return cudaGetLastError();
}

}  // namespace gspec
