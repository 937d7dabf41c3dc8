// batch.cu — stream-level batching (Alg. 1 L2-3 "for each input
// stream"): many independent streams of one DFA in one call.
//
// Every stream s is split into chunks of B bytes (its last chunk may be short).
// K1 runs every chunk of every stream speculatively: a stream's first chunk
// starts at q0 (exact), any other chunk at the top-ranked lookback-2 candidate
// (P:300).  K2 then walks each stream's chain of chunk records with one thread
// per stream: a record whose start equals the verified incoming state is taken
// as is (Alg. 2 L7-8), a mispredicted chunk is re-executed on the spot from the
// verified state (the paper's sequential recovery, Alg. 2 L9-11) with path
// fusion against the chunk's speculative path ([21]).  Streams are
// independent, so the recoveries of different streams run in parallel; within a
// stream the chain is exact by construction.
#include <algorithm>

#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr uint32_t kFuse = 256;  // bytes walked in lockstep with the recorded path

// chunk -> stream map: one thread per stream writes its id over its chunk range
__global__ void k_batch_map(const uint64_t* __restrict__ cbase, uint32_t ns, uint32_t* __restrict__ cs) {
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < ns; s += gridDim.x * blockDim.x)
    for (uint64_t c = __ldg(cbase + s), e = __ldg(cbase + s + 1); c < e; c++) cs[c] = s;
}

template <int MODE>
__global__ void __launch_bounds__(256) k_batch_spec(DevImage img, const uint8_t* __restrict__ in,
                                                   const uint64_t* __restrict__ off, const uint64_t* __restrict__ cbase,
                                                   const uint32_t* __restrict__ cs, uint64_t N, uint32_t B,
                                                   uint32_t q0t, uint32_t* __restrict__ rstart,
                                                   uint32_t* __restrict__ rend, uint32_t* __restrict__ rcnt) {
  extern __shared__ __align__(1024) uint8_t smem[];
  stage_table(img, smem);
  __syncthreads();
  using S = Step<MODE>;
  // P chunks per thread (P*g .. P*g+P-1), walked interleaved for ILP.  P = 2 pays for the
  // u8 table (one LDS per symbol, latency-bound lanes); the classed tables take 2-3 LDS
  // per symbol and a larger smem image (fewer resident CTAs): there one chunk per thread
  // is faster (measured on C3/C4 batches: 6.50 -> 5.83 ms, 2.94 -> 2.08 ms).
  constexpr int P = MODE == MODE_U8 ? 2 : 1;
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; P * g < N; g += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t lo[P], hi[P];
    uint32_t st[P], code[P], acc[P];
#pragma unroll
    for (int i = 0; i < P; i++) {
      const uint64_t c = min(P * g + i, N - 1);  // odd N: the last thread walks its chunk twice
      const uint32_t s = __ldg(cs + c);
      const uint64_t k = c - __ldg(cbase + s);
      lo[i] = __ldg(off + s) + k * B;
      hi[i] = min(lo[i] + B, __ldg(off + s + 1));
      st[i] = q0t;
      if (k > 0) {  // lookback-2 over the previous chunk's last two bytes (same stream, B >= 16)
        const uint32_t pair =
            (uint32_t)__ldg(img.cls + __ldg(in + lo[i] - 2)) * img.C + __ldg(img.cls + __ldg(in + lo[i] - 1));
        st[i] = __ldg(img.qs2 + (uint64_t)pair * kQsMax);
      }
      code[i] = __ldg(img.tid2code + st[i]);
      acc[i] = 0;
    }
    if constexpr (P == 2)
      walk2_bytes<MODE>(img, smem, in + lo[0], hi[0] - lo[0], code[0], acc[0], in + lo[1], hi[1] - lo[1], code[1],
                        acc[1]);
    else
      code[0] = walk_bytes<MODE>(img, smem, in + lo[0], hi[0] - lo[0], code[0], acc[0]);
#pragma unroll
    for (int i = 0; i < P; i++) {
      const uint64_t c = P * g + i;
      if (c >= N) break;
      rstart[c] = st[i];
      rend[c] = S::tid(img, code[i]);
      rcnt[c] = acc[i];
    }
  }
}

// Re-execute chunk [p, p+n) from `start`, in lockstep with the recorded path from
// `rstart` (end rend, count rcnt) until the two coincide (DFA determinism: the rest
// of the path is the recorded one).
template <int MODE>
__device__ void fused_walk(const DevImage& img, const uint8_t* smem, const uint8_t* p, uint64_t n, uint32_t start,
                           uint32_t rstart, uint32_t rend, uint32_t rcnt, uint32_t* end_out, uint32_t* cnt_out) {
  using S = Step<MODE>;
  uint32_t code = __ldg(img.tid2code + start), rcode = __ldg(img.tid2code + rstart);
  uint32_t acc = 0, racc = 0;
  uint64_t i = 0;
  // unaligned head: both paths byte by byte up to the 16-byte boundary
  const uint64_t head = min(n, (uint64_t)((16u - (reinterpret_cast<uintptr_t>(p) & 15u)) & 15u));
  for (; i < head; i++) {
    const uint32_t b = __ldg(p + i);
    code = S::byte(img, smem, code, b); acc += S::acc(code);
    rcode = S::byte(img, smem, rcode, b); racc += S::acc(rcode);
  }
  if (head && code == rcode) {
    *end_out = rend;
    *cnt_out = rcnt - racc + acc;
    return;
  }
  p += head;
  n -= head;
  i = 0;
  {
    const uint64_t nf = min(n, (uint64_t)kFuse) / 16;
    const uint4* v = reinterpret_cast<const uint4*>(p);
    for (uint64_t j = 0; j < nf; j++) {
      const uint4 q = __ldg(v + j);
      const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
      for (int t = 0; t < 4; t++) {
        code = S::template word<0>(img, smem, code, w[t]); acc += S::acc(code);
        rcode = S::template word<0>(img, smem, rcode, w[t]); racc += S::acc(rcode);
        code = S::template word<1>(img, smem, code, w[t]); acc += S::acc(code);
        rcode = S::template word<1>(img, smem, rcode, w[t]); racc += S::acc(rcode);
        code = S::template word<2>(img, smem, code, w[t]); acc += S::acc(code);
        rcode = S::template word<2>(img, smem, rcode, w[t]); racc += S::acc(rcode);
        code = S::template word<3>(img, smem, code, w[t]); acc += S::acc(code);
        rcode = S::template word<3>(img, smem, rcode, w[t]); racc += S::acc(rcode);
      }
      if (code == rcode) {
        *end_out = rend;
        *cnt_out = rcnt - racc + acc;
        return;
      }
    }
    i = nf * 16;
  }
  code = walk_bytes<MODE>(img, smem, p + i, n - i, code, acc);
  *end_out = S::tid(img, code);
  *cnt_out = acc;
}

struct BatchTotals {
  unsigned long long recoveries, reread, invalid;
};

template <int MODE>
__global__ void __launch_bounds__(128) k_batch_chain(DevImage img, const uint8_t* __restrict__ in,
                                                    const uint64_t* __restrict__ off,
                                                    const uint64_t* __restrict__ cbase, uint32_t ns, uint32_t B,
                                                    uint32_t q0t, const uint32_t* __restrict__ rstart,
                                                    const uint32_t* __restrict__ rend,
                                                    const uint32_t* __restrict__ rcnt, uint32_t* __restrict__ fin,
                                                    unsigned long long* __restrict__ count,
                                                    uint32_t* __restrict__ chunk_ends, BatchTotals* tot) {
  extern __shared__ __align__(1024) uint8_t smem[];
  stage_table(img, smem);
  __syncthreads();
  unsigned long long rec = 0, reread = 0, bad = 0;
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < ns; s += gridDim.x * blockDim.x) {
    const uint64_t c0 = __ldg(cbase + s), c1 = __ldg(cbase + s + 1), o = __ldg(off + s), oe = __ldg(off + s + 1);
    uint32_t x = q0t;
    unsigned long long cnt = 0;
    constexpr int kU = 8;  // records of kU chunks loaded before the chain consumes them
    for (uint64_t cb = c0; cb < c1; cb += kU) {
      uint32_t a[kU], e[kU], k[kU];
#pragma unroll
      for (int u = 0; u < kU; u++) {
        const uint64_t c = min(cb + u, c1 - 1);
        a[u] = __ldg(rstart + c);
        e[u] = __ldg(rend + c);
        k[u] = __ldg(rcnt + c);
      }
#pragma unroll
      for (int u = 0; u < kU; u++) {
        const uint64_t c = cb + u;
        if (c >= c1) break;
        if (a[u] == x) {  // speculation verified (Alg. 2 L7-8)
          x = e[u];
          cnt += k[u];
        } else {          // mispredicted: re-execute from the verified state (Alg. 2 L9-11)
          const uint64_t lo = o + (c - c0) * B, hi = min(lo + B, oe);
          uint32_t e2, k2;
          fused_walk<MODE>(img, smem, in + lo, hi - lo, x, a[u], e[u], k[u], &e2, &k2);
          x = e2;
          cnt += k2;
          rec++;
          reread += hi - lo;
        }
        if (chunk_ends) chunk_ends[c] = __ldg(img.inv + x);
      }
    }
    fin[s] = __ldg(img.inv + x);  // poison -> nstates: an input byte >= nsyms (R4)
    count[s] = cnt;
    bad += x == img.n;
  }
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    rec += __shfl_down_sync(0xffffffffu, rec, d);
    reread += __shfl_down_sync(0xffffffffu, reread, d);
    bad += __shfl_down_sync(0xffffffffu, bad, d);
  }
  if ((threadIdx.x & 31) == 0) {
    if (rec) atomicAdd(&tot->recoveries, rec);
    if (reread) atomicAdd(&tot->reread, reread);
    if (bad) atomicAdd(&tot->invalid, bad);
  }
}

template <int MODE>
cudaError_t launch_batch_m(const DevImage& img, const uint8_t* in, const uint64_t* off, const uint64_t* cbase,
                           uint32_t ns, uint64_t N, uint32_t B, uint32_t* cs, uint32_t* rs, uint32_t* re, uint32_t* rc,
                           uint32_t* fin, unsigned long long* count, uint32_t* chunk_ends, void* tot,
                           cudaStream_t st, int sms) {
  const uint32_t smem = smem_bytes_for(img);
  auto k1 = k_batch_spec<MODE>;
  auto k2 = k_batch_chain<MODE>;
  int occ = 0;
  cudaError_t e = kernel_setup((const void*)k1, smem, 256, &occ);
  if (e != cudaSuccess) return e;
  if (N > 0) {
    k_batch_map<<<(unsigned)std::min<uint64_t>((ns + 255) / 256, (uint64_t)sms * 8), 256, 0, st>>>(cbase, ns, cs);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    const uint64_t per = MODE == MODE_U8 ? 2 : 1;  // chunks per thread (k_batch_spec's P)
    uint64_t grid = std::min<uint64_t>((N / per + 256) / 256, (uint64_t)sms * std::max(occ, 1));
    k1<<<(unsigned)std::max<uint64_t>(grid, 1), 256, smem, st>>>(img, in, off, cbase, cs, N, B, img.q0t, rs, re, rc);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  if ((e = kernel_setup((const void*)k2, smem, 128, &occ)) != cudaSuccess) return e;
  uint64_t grid2 = std::min<uint64_t>((ns + 127) / 128, (uint64_t)sms * std::max(occ, 1));
  k2<<<(unsigned)std::max<uint64_t>(grid2, 1), 128, smem, st>>>(img, in, off, cbase, ns, B, img.q0t, rs, re, rc, fin,
                                                               count, chunk_ends,
                                                               reinterpret_cast<BatchTotals*>(tot));
  return cudaGetLastError();
}

}  // namespace

uint64_t batch_totals_bytes() { return sizeof(BatchTotals); }

cudaError_t launch_batch(const DevImage& img, const uint8_t* in, const uint64_t* off, const uint64_t* cbase,
                         uint32_t ns, uint64_t N, uint32_t B, uint32_t* cs, uint32_t* rs, uint32_t* re, uint32_t* rc,
                         uint32_t* fin,
                         unsigned long long* count, uint32_t* chunk_ends, void* tot, cudaStream_t st, int sms) {
  switch (img.mode) {
    case MODE_U8: return launch_batch_m<MODE_U8>(img, in, off, cbase, ns, N, B, cs, rs, re, rc, fin, count, chunk_ends, tot, st, sms);
    case MODE_U16: return launch_batch_m<MODE_U16>(img, in, off, cbase, ns, N, B, cs, rs, re, rc, fin, count, chunk_ends, tot, st, sms);
    case MODE_U16H: return launch_batch_m<MODE_U16H>(img, in, off, cbase, ns, N, B, cs, rs, re, rc, fin, count, chunk_ends, tot, st, sms);
    case MODE_U16D: return launch_batch_m<MODE_U16D>(img, in, off, cbase, ns, N, B, cs, rs, re, rc, fin, count, chunk_ends, tot, st, sms);
    default: return launch_batch_m<MODE_U32>(img, in, off, cbase, ns, N, B, cs, rs, re, rc, fin, count, chunk_ends, tot, st, sms);
  }
}

}  // namespace gspec
