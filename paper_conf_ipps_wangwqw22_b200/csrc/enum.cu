// enum.cu — B5: the enumerative scheme (Mytkowicz et al. [23]).
//
// Every sub-chunk j (E bytes, E | B) is run from EVERY transformed state
// (n+1 <= 64 incl. poison): M_j[q] = end state, C_j[q] = accepts on that path.
// Maps are W = 32 or 64 entries wide (W = 64: lane l of a warp holds entries l and l+32).
// The real path is obtained by "connecting the end state of each chunk to the
// start state of its successor", i.e. a prefix composition of maps:
//   (M2,C2) o (M1,C1) = (M2[M1[q]], C1[q] + C2[M1[q]]).
// Composition is one __shfl_sync per map (lane q holds entry q; two for W = 64), applied as a
// hierarchical scan: warps scan groups of 64 maps, group totals form the next
// level, the top level (<= 64 maps) is scanned by one warp, and incoming
// states/counts are pushed back down level by level.
#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr uint32_t kGroup = 64;

// The 16-byte-aligned vectors of [p, p+n) through TK, NE chains: codes are TK
// row offsets (tid * kTkRow) on entry; a vector holding a byte TK does not cover goes one
// symbol at a time through the transformed table.  On return the codes are table codes again
// and the result is the number of bytes consumed (0 when p is not 16-byte aligned).
template <int MODE, int NE>
__device__ __forceinline__ uint64_t tk_walk(const DevImage& img, const uint8_t* smem, uint32_t tkbase, uint32_t K,
                                            const uint8_t* p, uint64_t n, uint32_t (&code)[NE], uint32_t (&acc)[NE]) {
  using S = Step<MODE>;
  uint64_t i = 0;
  // packed maps (img.pk_off, K = 8, nt <= 8): code[] holds tids inside the vector loop
  const bool pk = NE == 8 && img.pk_off != 0;
  const uint32_t pkbase = tkbase + img.pk_off;
  if (pk) {
#pragma unroll
    for (int q = 0; q < NE; q++) code[q] /= kTkRow;
  }
  if ((reinterpret_cast<uintptr_t>(p) & 15u) == 0) {
    const uint4* v = reinterpret_cast<const uint4*>(p);
    const uint64_t nv = n / 16;
    // the lookups are cheap now: keep PF 16-byte loads in flight ahead of them
    constexpr int PF = NE <= 16 ? 4 : 1;
    uint4 buf[PF];
#pragma unroll
    for (int k = 0; k < PF; k++) buf[k] = (uint64_t)k < nv ? __ldg(v + k) : make_uint4(0, 0, 0, 0);
    for (uint64_t g0 = 0; g0 < nv; g0 += PF) {
      uint4 cur[PF];
#pragma unroll
      for (int k = 0; k < PF; k++) {
        cur[k] = buf[k];
        buf[k] = g0 + PF + k < nv ? __ldg(v + g0 + PF + k) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int k = 0; k < PF; k++) {
        const uint64_t t16 = g0 + k;
        if (t16 >= nv) break;
        const uint4 qv = cur[k];
        if (tk_vector_ok(qv, K)) {
          if (pk)
            pk_vector<NE>(pkbase, qv, code, acc);
          else
            tk_vector<NE>(tkbase, K, qv, code, acc);
        } else {  // a byte TK does not cover (an invalid symbol): these 16 bytes one by one
#pragma unroll
          for (int q = 0; q < NE; q++) code[q] = __ldg(img.tid2code + (pk ? code[q] : code[q] / kTkRow));
          const uint8_t* b16 = reinterpret_cast<const uint8_t*>(v + t16);
          for (int b = 0; b < 16; b++) {
            const uint32_t bb = __ldg(b16 + b);
#pragma unroll
            for (int q = 0; q < NE; q++) { code[q] = S::byte(img, smem, code[q], bb); acc[q] += S::acc(code[q]); }
          }
#pragma unroll
          for (int q = 0; q < NE; q++) code[q] = S::tid(img, code[q]) * (pk ? 1u : kTkRow);
        }
      }
    }
    i = nv * 16;
  }
#pragma unroll
  for (int q = 0; q < NE; q++) code[q] = __ldg(img.tid2code + (pk ? code[q] : code[q] / kTkRow));
  return i;
}

// K1: thread per sub-chunk, NE independent chains (ILP = NE).  SUPER: the 16-byte vectors
// whose bytes are all symbols TK covers advance K symbols per lookup (walk.cuh); any other
// byte (and the unaligned head / the tail) takes the one-symbol step of the transformed table.
template <int MODE, int NE, int W, bool SUPER = false>
__global__ void __launch_bounds__(128) k_enum_walk(DevImage img, const uint8_t* __restrict__ in, uint64_t len,
                                                  uint32_t E, uint64_t nsub, uint8_t* __restrict__ M,
                                                  uint64_t* __restrict__ Cn, Ctl* ctl_init, uint32_t q0t, uint64_t N) {
  extern __shared__ __align__(1024) uint8_t smem[];
  if (ctl_init && blockIdx.x == 0) init_ctl(ctl_init, q0t, N);  // the run's control block (no H2D copy)
  stage_table(img, smem);
  if (SUPER) {
    const uint4* src = reinterpret_cast<const uint4*>(img.TK);
    uint4* dst = reinterpret_cast<uint4*>(smem + tk_off(img));
    for (uint32_t i = threadIdx.x; i < img.tk_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  using S = Step<MODE>;
  const uint32_t nt = img.n + 1;
  const uint32_t tkbase = static_cast<uint32_t>(__cvta_generic_to_shared(smem)) + tk_off(img);
  const uint32_t K = img.tk_syms;
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < nsub; j += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t code[NE], acc[NE];
#pragma unroll
    for (int q = 0; q < NE; q++) {
      code[q] = SUPER ? ((uint32_t)q < nt ? q : 0) * kTkRow : __ldg(img.tid2code + ((uint32_t)q < nt ? q : 0));
      acc[q] = 0;
    }
    const uint64_t lo = j * E, n = min((uint64_t)E, len - lo);
    const uint8_t* p = in + lo;
    uint64_t i = 0;
    if (SUPER) {  // codes are TK row offsets until tk_walk returns
      i = tk_walk<MODE, NE>(img, smem, tkbase, K, p, n, code, acc);
    } else if ((reinterpret_cast<uintptr_t>(p) & 15u) == 0) {
      const uint4* v = reinterpret_cast<const uint4*>(p);
      for (uint64_t t16 = 0; t16 < n / 16; t16++) {
        const uint4 qv = __ldg(v + t16);
        const uint32_t w[4] = {qv.x, qv.y, qv.z, qv.w};
#pragma unroll
        for (int t = 0; t < 4; t++) {
#pragma unroll
          for (int q = 0; q < NE; q++) { code[q] = S::template word<0>(img, smem, code[q], w[t]); acc[q] += S::acc(code[q]); }
#pragma unroll
          for (int q = 0; q < NE; q++) { code[q] = S::template word<1>(img, smem, code[q], w[t]); acc[q] += S::acc(code[q]); }
#pragma unroll
          for (int q = 0; q < NE; q++) { code[q] = S::template word<2>(img, smem, code[q], w[t]); acc[q] += S::acc(code[q]); }
#pragma unroll
          for (int q = 0; q < NE; q++) { code[q] = S::template word<3>(img, smem, code[q], w[t]); acc[q] += S::acc(code[q]); }
        }
      }
      i = (n / 16) * 16;
    }
    for (; i < n; i++) {
      const uint32_t bb = __ldg(p + i);
#pragma unroll
      for (int q = 0; q < NE; q++) { code[q] = S::byte(img, smem, code[q], bb); acc[q] += S::acc(code[q]); }
    }
#pragma unroll
    for (int q = 0; q < W; q++) {
      const bool real = q < NE && (uint32_t)q < nt;
      M[j * W + q] = (uint8_t)(real ? S::tid(img, code[q < NE ? q : 0]) : q);
      Cn[j * W + q] = real ? acc[q < NE ? q : 0] : 0;
    }
  }
}

// One composition step P <- M o P for a W-entry map held by a warp: lane l owns entries l
// (and l + 32 when W = 64); m_lo / m_hi are this lane's entries of M.
template <int W>
__device__ __forceinline__ void compose_step(uint32_t& P0, uint32_t& P1, uint64_t& C0, uint64_t& C1, uint32_t m_lo,
                                             uint32_t m_hi, uint64_t c_lo, uint64_t c_hi) {
  if (W == 32) {
    const uint32_t nP = __shfl_sync(0xffffffffu, m_lo, P0);
    C0 += __shfl_sync(0xffffffffu, c_lo, P0);
    P0 = nP;
  } else {
    const uint32_t a0 = __shfl_sync(0xffffffffu, m_lo, P0 & 31), b0 = __shfl_sync(0xffffffffu, m_hi, P0 & 31);
    const uint64_t ca0 = __shfl_sync(0xffffffffu, c_lo, P0 & 31), cb0 = __shfl_sync(0xffffffffu, c_hi, P0 & 31);
    const uint32_t a1 = __shfl_sync(0xffffffffu, m_lo, P1 & 31), b1 = __shfl_sync(0xffffffffu, m_hi, P1 & 31);
    const uint64_t ca1 = __shfl_sync(0xffffffffu, c_lo, P1 & 31), cb1 = __shfl_sync(0xffffffffu, c_hi, P1 & 31);
    C0 += P0 < 32 ? ca0 : cb0;
    C1 += P1 < 32 ? ca1 : cb1;
    P0 = P0 < 32 ? a0 : b0;
    P1 = P1 < 32 ? a1 : b1;
  }
}

// K2: warp per group of kGroup maps: in-place inclusive prefix P_j = M_j o ... o M_g0,
// and the group total written as one map of the next level.  The maps are loaded in
// batches of kBatch (independent loads in flight) before the dependent shuffle chain
// consumes them, so a group costs kGroup / kBatch memory round trips, not kGroup.
constexpr int kBatch = 8;
template <int W>
__global__ void __launch_bounds__(128) k_enum_group(uint8_t* __restrict__ M, uint64_t* __restrict__ Cn, uint64_t cnt,
                                                   uint8_t* __restrict__ Mup, uint64_t* __restrict__ Cup) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t ngroups = (cnt + kGroup - 1) / kGroup;
  for (uint64_t g = warp; g < ngroups; g += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    uint32_t P0 = lane, P1 = lane + 32;
    uint64_t C0 = 0, C1 = 0;
    const uint64_t j0 = g * kGroup, j1 = min(cnt, j0 + kGroup);
    for (uint64_t jb = j0; jb < j1; jb += kBatch) {
      uint32_t m0[kBatch], m1[kBatch];
      uint64_t c0[kBatch], c1[kBatch];
#pragma unroll
      for (int u = 0; u < kBatch; u++) {
        const uint64_t j = min(jb + u, j1 - 1);
        m0[u] = M[j * W + lane];
        c0[u] = Cn[j * W + lane];
        m1[u] = W == 64 ? M[j * W + 32 + lane] : 0u;
        c1[u] = W == 64 ? Cn[j * W + 32 + lane] : 0ull;
      }
#pragma unroll
      for (int u = 0; u < kBatch; u++) {
        if (jb + u >= j1) break;
        compose_step<W>(P0, P1, C0, C1, m0[u], m1[u], c0[u], c1[u]);
        M[(jb + u) * W + lane] = (uint8_t)P0;
        Cn[(jb + u) * W + lane] = C0;
        if (W == 64) {
          M[(jb + u) * W + 32 + lane] = (uint8_t)P1;
          Cn[(jb + u) * W + 32 + lane] = C1;
        }
      }
    }
    if (Mup) {
      Mup[g * W + lane] = (uint8_t)P0;
      Cup[g * W + lane] = C0;
      if (W == 64) {
        Mup[g * W + 32 + lane] = (uint8_t)P1;
        Cup[g * W + 32 + lane] = C1;
      }
    }
  }
}

// Descend: incoming state/count of every map at level l from its group's entry.
template <int W>
__global__ void k_enum_descend(const uint8_t* __restrict__ P, const uint64_t* __restrict__ PC, uint64_t cnt,
                               const uint32_t* __restrict__ up_state, const uint64_t* __restrict__ up_cnt,
                               uint32_t top_entry, uint32_t* __restrict__ st, uint64_t* __restrict__ sc) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < cnt; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t g = j / kGroup;
    const uint32_t e = up_state ? up_state[g] : top_entry;
    const uint64_t ec = up_state ? up_cnt[g] : 0;
    if (j % kGroup == 0) {
      st[j] = e;
      sc[j] = ec;
    } else {
      st[j] = P[(j - 1) * W + e];
      sc[j] = ec + PC[(j - 1) * W + e];
    }
  }
}

// Outputs: chunk ends (original ids), final state (transformed), total count.
template <int W>
__global__ void k_enum_out(DevImage img, const uint32_t* __restrict__ st0, const uint8_t* __restrict__ P0top,
                           const uint64_t* __restrict__ PC0top, uint64_t top_last, uint32_t q0t, uint64_t nsub,
                           uint32_t per_chunk, uint64_t N, uint32_t* __restrict__ chunk_ends, Ctl* ctl,
                           uint32_t* __restrict__ x_final, void* h_out) {
  const uint32_t fin = P0top[top_last * W + q0t];
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < N; c += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t jn = (c + 1) * per_chunk;  // first sub-chunk after chunk c
    const uint32_t s = jn < nsub ? st0[jn] : fin;
    if (chunk_ends) chunk_ends[c] = img.inv[s];
  }
  if (blockIdx.x == 0) {
    if (threadIdx.x == 0) {
      *x_final = fin;
      ctl->accept_count = PC0top[top_last * W + q0t];
      __threadfence();
    }
    __syncthreads();
    if (h_out) {  // zero-copy result: the block publishes the control block to the pinned host slot
      const uint32_t* src = reinterpret_cast<const uint32_t*>(ctl);
      uint32_t* dst = reinterpret_cast<uint32_t*>(h_out);
      for (uint32_t i = threadIdx.x; i < sizeof(Ctl) / 4; i += blockDim.x) dst[i] = __ldcg(src + i);
    }
  }
}

template <int MODE, int NE, int W, bool SUPER = false>
cudaError_t walk_t(const DevImage& img, const RunParams& rp, uint32_t E, uint64_t nsub, uint8_t* M, uint64_t* Cn,
                   cudaStream_t st, int sms) {
  auto kern = k_enum_walk<MODE, NE, W, SUPER>;
  const uint32_t smem = SUPER ? tk_off(img) + img.tk_bytes : smem_bytes_for(img);
  cudaError_t e = kernel_setup((const void*)kern, smem, 128, nullptr);
  if (e != cudaSuccess) return e;
  uint64_t grid = (nsub + 127) / 128;
  const uint64_t cap = (uint64_t)sms * 16;
  if (grid > cap) grid = cap;
  kern<<<(unsigned)grid, 128, smem, st>>>(img, rp.in, rp.len, E, nsub, M, Cn, rp.ctl_init, rp.q0t, rp.N);
  return cudaGetLastError();
}

template <int MODE>
cudaError_t walk_m(const DevImage& img, const RunParams& rp, uint32_t E, uint64_t nsub, uint8_t* M, uint64_t* Cn,
                   cudaStream_t st, int sms) {
  const uint32_t nt = img.n + 1;
  if (MODE == MODE_U8 && img.TK && !tk_disabled()) {  // small alphabet: K symbols per lookup
    if (nt <= 8) return walk_t<MODE, 8, 32, true>(img, rp, E, nsub, M, Cn, st, sms);
    if (nt <= 16) return walk_t<MODE, 16, 32, true>(img, rp, E, nsub, M, Cn, st, sms);
    if (nt <= 32) return walk_t<MODE, 32, 32, true>(img, rp, E, nsub, M, Cn, st, sms);
    return walk_t<MODE, 64, 64, true>(img, rp, E, nsub, M, Cn, st, sms);
  }
  if (nt <= 8) return walk_t<MODE, 8, 32>(img, rp, E, nsub, M, Cn, st, sms);
  if (nt <= 16) return walk_t<MODE, 16, 32>(img, rp, E, nsub, M, Cn, st, sms);
  if (nt <= 32) return walk_t<MODE, 32, 32>(img, rp, E, nsub, M, Cn, st, sms);
  return walk_t<MODE, 64, 64>(img, rp, E, nsub, M, Cn, st, sms);
}

// ---- small streams: the whole enumeration in ONE launch -------------------------
// K1+K2+descend+outputs fused for nsub <= kSmallCTAs * kSmallT sub-chunks: each CTA walks
// kSmallT sub-chunks (one per thread, NE chains), one warp scans the CTA's maps in shared
// memory (lane q holds entry q; a composition is one shuffle), the CTA publishes
// its aggregate map, and the last CTA to finish (ticket) composes the aggregates from q0,
// writes every chunk end, the accept count and the control block (zero-copy to the host).
constexpr int kSmallT = 128;
constexpr int kSmallCTAs = 64;

template <int MODE, int NE, bool SUPER = false>
__global__ void __launch_bounds__(kSmallT) k_enum_small(DevImage img, RunParams rp, uint32_t E, uint64_t nsub,
                                                       uint8_t* __restrict__ P, uint64_t* __restrict__ PC,
                                                       uint8_t* __restrict__ AM, uint64_t* __restrict__ AC,
                                                       uint32_t* __restrict__ ticket, uint32_t* __restrict__ chunk_ends,
                                                       Ctl* ctl) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint8_t sM[kSmallT][33];  // +1 pad: a thread's 32 writes of its own map hit
  __shared__ unsigned long long sC[kSmallT][33];  // different banks from its neighbours' writes
  __shared__ uint8_t s_in[kSmallCTAs];
  __shared__ uint32_t last;
  if (rp.ctl_init && blockIdx.x == 0) init_ctl(rp.ctl_init, rp.q0t, rp.N);
  stage_table(img, smem);
  if (SUPER) {
    const uint4* src = reinterpret_cast<const uint4*>(img.TK);
    uint4* dst = reinterpret_cast<uint4*>(smem + tk_off(img));
    for (uint32_t i = threadIdx.x; i < img.tk_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  using S = Step<MODE>;
  const uint32_t nt = img.n + 1, t = threadIdx.x;
  const uint64_t j = (uint64_t)blockIdx.x * kSmallT + t;
  {  // walk sub-chunk j from every state (ILP = NE chains)
    uint32_t code[NE], acc[NE];
#pragma unroll
    for (int q = 0; q < NE; q++) {
      code[q] = SUPER ? ((uint32_t)q < nt ? q : 0) * kTkRow : __ldg(img.tid2code + ((uint32_t)q < nt ? q : 0));
      acc[q] = 0;
    }
    if (SUPER && j >= nsub) {
#pragma unroll
      for (int q = 0; q < NE; q++) code[q] = __ldg(img.tid2code + code[q] / kTkRow);
    }
    if (j < nsub) {
      const uint64_t lo = j * E, n = min((uint64_t)E, rp.len - lo);
      const uint8_t* p = rp.in + lo;
      const uint4* v = reinterpret_cast<const uint4*>(p);
      uint64_t i = 0;
      if (SUPER) {
        i = tk_walk<MODE, NE>(img, smem, static_cast<uint32_t>(__cvta_generic_to_shared(smem)) + tk_off(img),
                              img.tk_syms, p, n, code, acc);
      } else if ((reinterpret_cast<uintptr_t>(p) & 15u) == 0) {
        for (uint64_t t16 = 0; t16 < n / 16; t16++) {
          const uint4 qv = __ldg(v + t16);
          const uint32_t w[4] = {qv.x, qv.y, qv.z, qv.w};
#pragma unroll
          for (int k = 0; k < 4; k++) {
#pragma unroll
            for (int q = 0; q < NE; q++) { code[q] = S::template word<0>(img, smem, code[q], w[k]); acc[q] += S::acc(code[q]); }
#pragma unroll
            for (int q = 0; q < NE; q++) { code[q] = S::template word<1>(img, smem, code[q], w[k]); acc[q] += S::acc(code[q]); }
#pragma unroll
            for (int q = 0; q < NE; q++) { code[q] = S::template word<2>(img, smem, code[q], w[k]); acc[q] += S::acc(code[q]); }
#pragma unroll
            for (int q = 0; q < NE; q++) { code[q] = S::template word<3>(img, smem, code[q], w[k]); acc[q] += S::acc(code[q]); }
          }
        }
        i = (n / 16) * 16;
      }
      for (; i < n; i++) {
        const uint32_t bb = __ldg(p + i);
#pragma unroll
        for (int q = 0; q < NE; q++) { code[q] = S::byte(img, smem, code[q], bb); acc[q] += S::acc(code[q]); }
      }
    }
#pragma unroll
    for (int q = 0; q < 32; q++) {
      const bool real = q < NE && (uint32_t)q < nt && j < nsub;
      sM[t][q] = (uint8_t)(real ? S::tid(img, code[q < NE ? q : 0]) : q);  // identity past the stream
      sC[t][q] = real ? acc[q < NE ? q : 0] : 0;
    }
  }
  __syncthreads();
  const uint64_t G = (nsub + kSmallT - 1) / kSmallT;
  if (t < 32) {  // in-CTA inclusive prefix: P_i = M_i o ... o M_0 (lane t holds entry t)
    uint32_t x = t;
    unsigned long long c = 0;
    for (int i = 0; i < kSmallT; i++) {
      const uint32_t y = __shfl_sync(0xffffffffu, (uint32_t)sM[i][t], x);
      c += __shfl_sync(0xffffffffu, sC[i][t], x);
      x = y;
      const uint64_t ji = (uint64_t)blockIdx.x * kSmallT + i;
      if (ji < nsub) {
        P[ji * 32 + t] = (uint8_t)x;
        PC[ji * 32 + t] = c;
      }
    }
    AM[blockIdx.x * 32 + t] = (uint8_t)x;
    AC[blockIdx.x * 32 + t] = c;
  }
  __threadfence();
  __syncthreads();
  if (t == 0) last = atomicAdd(ticket, 1u) == G - 1;
  __syncthreads();
  if (!last) return;
  __threadfence();
  // the CTA aggregates into shared memory first (independent loads), then the dependent
  // composition chain runs on shared memory instead of G dependent L2 round trips
  for (uint32_t i = t; i < G * 32; i += kSmallT) {
    sM[i / 32][i % 32] = __ldcg(AM + i);
    sC[i / 32][i % 32] = __ldcg(reinterpret_cast<const unsigned long long*>(AC) + i);
  }
  __syncthreads();
  if (t < 32) {  // compose the CTA aggregates from q0: incoming state of every CTA
    uint32_t s = rp.q0t;
    unsigned long long total = 0;
    for (uint64_t g = 0; g < G; g++) {
      if (t == 0) s_in[g] = (uint8_t)s;
      total += sC[g][s];
      s = sM[g][s];
    }
    if (t == 0) {
      ctl->accept_count = total;
      ctl->xfin = s;
      *ticket = 0;  // re-armed for the next run
    }
  }
  __syncthreads();
  const uint32_t per = rp.B / E;  // sub-chunks per chunk
  for (uint64_t c = t; c < rp.N; c += kSmallT) {
    const uint64_t jl = min((c + 1) * per, nsub) - 1;
    const uint32_t sin = s_in[jl / kSmallT];
    if (chunk_ends) chunk_ends[c] = __ldg(img.inv + __ldcg(P + jl * 32 + sin));
  }
  if (t == 0) ctl->finished = 1;
  __threadfence();
  __syncthreads();
  if (rp.h_out) {  // zero-copy result, copied by the whole CTA (one thread would serialise ~130 L2 loads)
    const uint32_t* src = reinterpret_cast<const uint32_t*>(ctl);
    uint32_t* dst = reinterpret_cast<uint32_t*>(rp.h_out);
    for (uint32_t i = t; i < sizeof(Ctl) / 4; i += kSmallT) dst[i] = __ldcg(src + i);
  }
}

template <int MODE, int NE, bool SUPER = false>
cudaError_t small_t(const DevImage& img, const RunParams& rp, uint32_t E, uint64_t nsub, void* scratch,
                    uint32_t* ticket, uint32_t* chunk_ends, Ctl* ctl, cudaStream_t st) {
  auto kern = k_enum_small<MODE, NE, SUPER>;
  const uint32_t smem = SUPER ? tk_off(img) + img.tk_bytes : smem_bytes_for(img);
  cudaError_t e = kernel_setup((const void*)kern, smem, kSmallT, nullptr);
  if (e != cudaSuccess) return e;
  uint8_t* p = reinterpret_cast<uint8_t*>(scratch);
  auto take = [&](uint64_t bytes) { uint8_t* r = p; p += (bytes + 255) & ~255ull; return r; };
  uint8_t* P = take(nsub * 32);
  uint64_t* PC = reinterpret_cast<uint64_t*>(take(nsub * 32 * 8));
  uint8_t* AM = take(kSmallCTAs * 32);
  uint64_t* AC = reinterpret_cast<uint64_t*>(take(kSmallCTAs * 32 * 8));
  const uint64_t G = (nsub + kSmallT - 1) / kSmallT;
  kern<<<(unsigned)G, kSmallT, smem, st>>>(img, rp, E, nsub, P, PC, AM, AC, ticket, chunk_ends, ctl);
  return cudaGetLastError();
}

template <int MODE>
cudaError_t small_m(const DevImage& img, const RunParams& rp, uint32_t E, uint64_t nsub, void* scratch,
                    uint32_t* ticket, uint32_t* chunk_ends, Ctl* ctl, cudaStream_t st) {
  const uint32_t nt = img.n + 1;  // <= 32 (the caller takes the multi-launch path for wider maps)
  if (MODE == MODE_U8 && img.TK && !tk_disabled()) {  // small alphabet: K symbols per lookup
    if (nt <= 8) return small_t<MODE, 8, true>(img, rp, E, nsub, scratch, ticket, chunk_ends, ctl, st);
    if (nt <= 16) return small_t<MODE, 16, true>(img, rp, E, nsub, scratch, ticket, chunk_ends, ctl, st);
    return small_t<MODE, 32, true>(img, rp, E, nsub, scratch, ticket, chunk_ends, ctl, st);
  }
  if (nt <= 8) return small_t<MODE, 8>(img, rp, E, nsub, scratch, ticket, chunk_ends, ctl, st);
  if (nt <= 16) return small_t<MODE, 16>(img, rp, E, nsub, scratch, ticket, chunk_ends, ctl, st);
  return small_t<MODE, 32>(img, rp, E, nsub, scratch, ticket, chunk_ends, ctl, st);
}

}  // namespace

uint64_t enum_small_max_sub() { return (uint64_t)kSmallCTAs * kSmallT; }

uint64_t enum_small_scratch_bytes(uint64_t nsub) {
  auto r = [](uint64_t b) { return (b + 255) & ~255ull; };
  return r(nsub * 32) + r(nsub * 32 * 8) + r(kSmallCTAs * 32) + r(kSmallCTAs * 32 * 8);
}

// `ticket` (device u32, zero before the first launch) counts finished CTAs; the last CTA
// re-arms it, so runs queued back to back on one stream reuse it.
cudaError_t launch_enum_small(const DevImage& img, const RunParams& rp, uint32_t E, void* scratch, uint32_t* ticket,
                              uint32_t* d_chunk_ends, Ctl* d_ctl, cudaStream_t st) {
  const uint64_t nsub = (rp.len + E - 1) / E;
  switch (img.mode) {
    case MODE_U8: return small_m<MODE_U8>(img, rp, E, nsub, scratch, ticket, d_chunk_ends, d_ctl, st);
    case MODE_U16: return small_m<MODE_U16>(img, rp, E, nsub, scratch, ticket, d_chunk_ends, d_ctl, st);
    case MODE_U16H: return small_m<MODE_U16H>(img, rp, E, nsub, scratch, ticket, d_chunk_ends, d_ctl, st);
    case MODE_U16D: return small_m<MODE_U16D>(img, rp, E, nsub, scratch, ticket, d_chunk_ends, d_ctl, st);
    default: return small_m<MODE_U32>(img, rp, E, nsub, scratch, ticket, d_chunk_ends, d_ctl, st);
  }
}

// Scratch layout for the enumeration (levels of maps + per-level states); maps of up to 64
// entries (the carve in launch_enum_full uses the DFA's width, 32 or 64).
uint64_t enum_scratch_bytes(uint64_t nsub) {
  auto r = [](uint64_t b) { return (b + 255) & ~255ull; };  // same rounding as the carve in launch_enum_full
  uint64_t tot = 0, cnt = nsub;
  for (int L = 0;; L++) {
    tot += r(cnt * 64) + r(cnt * 64 * 8) + r(cnt * 4) + r(cnt * 8);
    if (cnt <= kGroup || L + 1 == 16) break;
    cnt = (cnt + kGroup - 1) / kGroup;
  }
  return tot + 1024;
}

// phases: 1 = start-independent part (walk + group scans); 2 = start-dependent
// part (descend from rp.q0t, outputs).  top_M/top_C (nullable) receive the
// device addresses of the whole-stream map and counts (entry q = from state q).
cudaError_t launch_enum_full(const DevImage& img, const RunParams& rp, uint32_t E, void* scratch,
                             uint32_t* d_chunk_ends, Ctl* d_ctl, uint32_t* d_x_final, cudaStream_t st, int sms,
                             int phases, const uint8_t** top_M, const uint64_t** top_C) {
  const uint64_t nsub = (rp.len + E - 1) / E;
  const uint32_t W = img.n + 1 <= 32 ? 32u : 64u;  // map width
  // carve levels
  struct Lvl { uint8_t* M; uint64_t* C; uint32_t* s; uint64_t* sc; uint64_t cnt; };
  Lvl lv[16];
  int L = 0;
  uint8_t* p = reinterpret_cast<uint8_t*>(scratch);
  auto take = [&](uint64_t bytes) { uint8_t* r = p; p += (bytes + 255) & ~255ull; return r; };
  uint64_t cnt = nsub;
  for (;;) {
    lv[L].cnt = cnt;
    lv[L].M = take(cnt * W);
    lv[L].C = reinterpret_cast<uint64_t*>(take(cnt * W * 8));
    lv[L].s = reinterpret_cast<uint32_t*>(take(cnt * 4));
    lv[L].sc = reinterpret_cast<uint64_t*>(take(cnt * 8));
    L++;
    if (cnt <= kGroup || L == 16) break;
    cnt = (cnt + kGroup - 1) / kGroup;
  }
  const uint64_t top_last = lv[L - 1].cnt - 1;
  if (top_M) *top_M = lv[L - 1].M + top_last * W;
  if (top_C) *top_C = lv[L - 1].C + top_last * W;
  cudaError_t e = cudaSuccess;
  if (phases & 1) {
  switch (img.mode) {
    case MODE_U8: e = walk_m<MODE_U8>(img, rp, E, nsub, lv[0].M, lv[0].C, st, sms); break;
    case MODE_U16: e = walk_m<MODE_U16>(img, rp, E, nsub, lv[0].M, lv[0].C, st, sms); break;
    case MODE_U16H: e = walk_m<MODE_U16H>(img, rp, E, nsub, lv[0].M, lv[0].C, st, sms); break;
    case MODE_U16D: e = walk_m<MODE_U16D>(img, rp, E, nsub, lv[0].M, lv[0].C, st, sms); break;
    default: e = walk_m<MODE_U32>(img, rp, E, nsub, lv[0].M, lv[0].C, st, sms); break;
  }
  if (e != cudaSuccess) return e;
  for (int l = 0; l < L; l++) {
    const uint64_t ng = (lv[l].cnt + kGroup - 1) / kGroup;
    uint64_t grid = (ng * 32 + 127) / 128;
    if (grid > (uint64_t)sms * 16) grid = (uint64_t)sms * 16;
    if (W == 32)
      k_enum_group<32><<<(unsigned)grid, 128, 0, st>>>(lv[l].M, lv[l].C, lv[l].cnt, l + 1 < L ? lv[l + 1].M : nullptr,
                                                       l + 1 < L ? lv[l + 1].C : nullptr);
    else
      k_enum_group<64><<<(unsigned)grid, 128, 0, st>>>(lv[l].M, lv[l].C, lv[l].cnt, l + 1 < L ? lv[l + 1].M : nullptr,
                                                       l + 1 < L ? lv[l + 1].C : nullptr);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  }
  if (!(phases & 2)) return cudaSuccess;
  for (int l = L - 1; l >= 0; l--) {
    uint64_t grid = (lv[l].cnt + 255) / 256;
    if (grid > (uint64_t)sms * 16) grid = (uint64_t)sms * 16;
    if (W == 32)
      k_enum_descend<32><<<(unsigned)grid, 256, 0, st>>>(lv[l].M, lv[l].C, lv[l].cnt,
                                                         l + 1 < L ? lv[l + 1].s : nullptr,
                                                         l + 1 < L ? lv[l + 1].sc : nullptr, rp.q0t, lv[l].s, lv[l].sc);
    else
      k_enum_descend<64><<<(unsigned)grid, 256, 0, st>>>(lv[l].M, lv[l].C, lv[l].cnt,
                                                         l + 1 < L ? lv[l + 1].s : nullptr,
                                                         l + 1 < L ? lv[l + 1].sc : nullptr, rp.q0t, lv[l].s, lv[l].sc);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  uint64_t grid = (rp.N + 255) / 256;
  if (grid > (uint64_t)sms * 16) grid = (uint64_t)sms * 16;
  if (grid < 1) grid = 1;
  if (W == 32)
    k_enum_out<32><<<(unsigned)grid, 256, 0, st>>>(img, lv[0].s, lv[L - 1].M, lv[L - 1].C, top_last, rp.q0t, nsub,
                                                   rp.B / E, rp.N, d_chunk_ends, d_ctl, d_x_final, rp.h_out);
  else
    k_enum_out<64><<<(unsigned)grid, 256, 0, st>>>(img, lv[0].s, lv[L - 1].M, lv[L - 1].C, top_last, rp.q0t, nsub,
                                                   rp.B / E, rp.N, d_chunk_ends, d_ctl, d_x_final, rp.h_out);
  return cudaGetLastError();
}

}  // namespace gspec
