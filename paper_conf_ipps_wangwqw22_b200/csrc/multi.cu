// multi.cu — FSM-level batching (second half; Alg. 1 L2-3 P:65-76:
// "Forall fsm in FSMs / Forall stream in streams"): many (DFA, input stream) pairs in
// ONE launch per table format.  One CTA owns one pair: it stages that DFA's transformed
// table in shared memory and runs the speculative method over the pair's stream in waves
// of 256 chunks — lookback-2 prediction and a walk per thread (Alg. 2 L3-6),
// then SRE rounds inside the CTA (Alg. 3's recovery from the predecessor's end)
// until every chunk's start equals its predecessor's end (the unique consistent chain).
// Convergent DFAs settle in one or two rounds; the CTA barrier replaces Alg. 3's sync().
#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr int kMT = 256;  // threads per CTA = chunks per wave

template <int MODE>
__global__ void __launch_bounds__(kMT) k_multi(const DevImage* __restrict__ imgs, const uint8_t* const* __restrict__ ins,
                                              const uint64_t* __restrict__ lens, const uint32_t* __restrict__ pairs,
                                              uint32_t B, uint32_t* __restrict__ fin_out,
                                              unsigned long long* __restrict__ cnt_out,
                                              unsigned long long* __restrict__ stats) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t s_end[kMT];
  __shared__ unsigned long long red[kMT / 32];
  using S = Step<MODE>;
  const uint32_t p = pairs[blockIdx.x];
  const DevImage img = imgs[p];
  stage_table(img, smem);
  const uint8_t* in = ins[p];
  const uint64_t len = lens[p];
  const uint64_t N = (len + B - 1) / B;
  const uint32_t t = threadIdx.x;
  uint32_t x_in = img.q0t;  // verified incoming state of the current wave
  unsigned long long total = 0, rewalks = 0, rounds = 0;
  __syncthreads();
  for (uint64_t w0 = 0; w0 < N; w0 += kMT) {
    const uint64_t c = w0 + t;
    const bool act = c < N;
    const uint64_t lo = c * B, n = act ? min((uint64_t)B, len - lo) : 0;
    auto walk = [&](uint32_t st, uint32_t* cnt) {  // FSM_Processing(fsm, Pi(c), st)
      uint32_t acc = 0;
      const uint32_t code = walk_bytes<MODE>(img, smem, in + lo, n, __ldg(img.tid2code + st), acc);
      *cnt = acc;
      return S::tid(img, code);
    };
    uint32_t st = x_in, e = x_in, cnt = 0;
    if (act) {
      if (c > 0) st = __ldg(img.qs2 + (uint64_t)qs_pair(img, in, c, B) * kQsMax);  // lookback-2
      e = walk(st, &cnt);
    }
    for (;;) {  // SRE rounds inside the wave
      s_end[t] = e;
      __syncthreads();
      const uint32_t inc = t == 0 ? x_in : s_end[t - 1];
      const bool redo = act && inc != st;
      __syncthreads();
      if (redo) {
        st = inc;
        e = walk(st, &cnt);
        rewalks++;
      }
      if (!__syncthreads_or(redo)) break;
      rounds += (t == 0);
    }
    total += act ? cnt : 0;
    const uint32_t last = (uint32_t)min((uint64_t)kMT, N - w0) - 1;
    s_end[t] = e;
    __syncthreads();
    x_in = s_end[last];
    __syncthreads();
  }
  // block sums: accept count, re-walks
  unsigned long long v[2] = {total, rewalks};
#pragma unroll
  for (int k = 0; k < 2; k++) {
    for (int o = 16; o > 0; o >>= 1) v[k] += __shfl_down_sync(0xffffffffu, v[k], o);
  }
  if ((t & 31) == 0) red[t >> 5] = v[0];
  __syncthreads();
  if (t == 0) {
    unsigned long long s = 0;
    for (int w = 0; w < kMT / 32; w++) s += red[w];
    cnt_out[p] = s;
    fin_out[p] = x_in == img.n ? 0xFFFFFFFFu : __ldg(img.inv + x_in);  // poison: an invalid symbol (R4)
    atomicAdd(stats + 1, rounds);
  }
  __syncthreads();
  if ((t & 31) == 0) red[t >> 5] = v[1];
  __syncthreads();
  if (t == 0) {
    unsigned long long s = 0;
    for (int w = 0; w < kMT / 32; w++) s += red[w];
    atomicAdd(stats, s);
  }
}

template <int MODE>
cudaError_t launch_multi_m(const DevImage* d_imgs, const uint8_t* const* d_ins, const uint64_t* d_lens,
                           const uint32_t* d_pairs, uint32_t npairs, uint32_t smem, uint32_t B, uint32_t* d_fin,
                           unsigned long long* d_cnt, unsigned long long* d_stats, cudaStream_t st) {
  auto kern = k_multi<MODE>;
  cudaError_t e = kernel_setup((const void*)kern, smem, kMT, nullptr);
  if (e != cudaSuccess) return e;
  kern<<<npairs, kMT, smem, st>>>(d_imgs, d_ins, d_lens, d_pairs, B, d_fin, d_cnt, d_stats);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_multi(int mode, const DevImage* d_imgs, const uint8_t* const* d_ins, const uint64_t* d_lens,
                         const uint32_t* d_pairs, uint32_t npairs, uint32_t smem, uint32_t B, uint32_t* d_fin,
                         unsigned long long* d_cnt, unsigned long long* d_stats, cudaStream_t st) {
  if (npairs == 0) return cudaSuccess;
  switch (mode) {
    case MODE_U8: return launch_multi_m<MODE_U8>(d_imgs, d_ins, d_lens, d_pairs, npairs, smem, B, d_fin, d_cnt, d_stats, st);
    case MODE_U16: return launch_multi_m<MODE_U16>(d_imgs, d_ins, d_lens, d_pairs, npairs, smem, B, d_fin, d_cnt, d_stats, st);
    case MODE_U16H: return launch_multi_m<MODE_U16H>(d_imgs, d_ins, d_lens, d_pairs, npairs, smem, B, d_fin, d_cnt, d_stats, st);
    case MODE_U16D: return launch_multi_m<MODE_U16D>(d_imgs, d_ins, d_lens, d_pairs, npairs, smem, B, d_fin, d_cnt, d_stats, st);
    default: return launch_multi_m<MODE_U32>(d_imgs, d_ins, d_lens, d_pairs, npairs, smem, B, d_fin, d_cnt, d_stats, st);
  }
}

}  // namespace gspec
