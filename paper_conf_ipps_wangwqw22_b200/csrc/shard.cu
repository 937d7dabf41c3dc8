// shard.cu — B8: multi-GPU contiguous sharding.
//
// Rank g owns a contiguous, chunk-aligned shard.  Its start state is unknown
// (g > 0), but it lies in the image of all states over the bytes just before
// the shard ("the real start state ... must be contained in the produced end
// state set").  Each rank enumerates that candidate set over its first
// chunks with path fusion (paths that meet stay merged), runs the normal
// speculative pipeline from the merge point, and publishes a state map over
// the transformed states; an allgather + composition fixes every start.
#include <algorithm>

#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr uint32_t kNoState = 0xFFFFFFFFu;

// candidate set: image of all real states over w[0..L) (L <= 16), compacted
// in increasing id order by one block.
__global__ void __launch_bounds__(1024) k_image(DevImage img, const uint32_t* __restrict__ ttc,
                                                const uint8_t* __restrict__ w, uint32_t L,
                                                uint32_t* __restrict__ mark, uint32_t* __restrict__ list,
                                                uint32_t* __restrict__ count) {
  const uint32_t nt = img.n + 1;
  __shared__ uint8_t cl[16];
  __shared__ uint32_t wsum[32];
  __shared__ uint32_t base;
  if (threadIdx.x < L) cl[threadIdx.x] = img.cls[w[threadIdx.x]];
  for (uint32_t s = threadIdx.x; s < nt; s += blockDim.x) mark[s] = 0;
  if (threadIdx.x == 0) base = 0;
  __syncthreads();
  for (uint32_t q = threadIdx.x; q < img.n; q += blockDim.x) {
    uint32_t t = q;
    for (uint32_t i = 0; i < L; i++) t = ttc[(uint64_t)t * img.C + cl[i]];
    mark[t] = 1;
  }
  __syncthreads();
  for (uint32_t t0 = 0; t0 < nt; t0 += blockDim.x) {
    const uint32_t s = t0 + threadIdx.x;
    const bool m = s < nt && mark[s];
    const uint32_t bal = __ballot_sync(0xffffffffu, m);
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (lane == 0) wsum[warp] = __popc(bal);
    __syncthreads();
    uint32_t off = base;
    for (uint32_t k = 0; k < warp; k++) off += wsum[k];
    if (m) list[off + __popc(bal & ((1u << lane) - 1))] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t tot = 0;
      for (uint32_t k = 0; k < blockDim.x / 32; k++) tot += wsum[k];
      base += tot;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) *count = base;
}

// Path fusion over whole chunks: thread i walks candidate i chunk by chunk and
// records its state at every chunk end; stop after the first chunk where all
// candidates coincide (info[0] = that chunk) or after max_chunks (info[0] =
// kNoState).  info[1] = chunks walked.
template <int MODE>
__global__ void __launch_bounds__(1024) k_fuse(DevImage img, const uint8_t* __restrict__ in, uint64_t len, uint32_t B,
                                               const uint32_t* __restrict__ cand, uint32_t ncand, uint32_t max_chunks,
                                               uint32_t* __restrict__ states, unsigned long long* __restrict__ cnt,
                                               uint32_t* __restrict__ info) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t s0;
  stage_table(img, smem);
  __syncthreads();
  using S = Step<MODE>;
  const uint32_t i = threadIdx.x;
  uint32_t code = i < ncand ? __ldg(img.tid2code + cand[i]) : 0;
  unsigned long long total = 0;
  const uint64_t N = (len + B - 1) / B;
  uint32_t merged = kNoState, j = 0;
  for (; j < max_chunks && j < N; j++) {
    const uint64_t lo = (uint64_t)j * B, n = min((uint64_t)B, len - lo);
    uint32_t acc = 0;
    if (i < ncand) code = walk_bytes<MODE>(img, smem, in + lo, n, code, acc);
    total += acc;
    const uint32_t t = S::tid(img, code);
    if (i < ncand) states[(uint64_t)j * ncand + i] = t;
    if (i == 0) s0 = t;
    __syncthreads();
    const bool same = __syncthreads_and(i >= ncand || t == s0);
    if (same) { merged = j; j++; break; }
  }
  if (i < ncand) cnt[i] = total;
  if (i == 0) { info[0] = merged; info[1] = j; }
}

// Path fusion against a reference candidate (cand[0]): thread i walks its
// candidate and the reference in lockstep, 16 bytes at a time, until the two
// states coincide (then the rest of the shard is shared, DFA determinism).
// merged[i] = chunk in which it merged (kNoState if not within max_chunks),
// dcnt[i] = accepts(own) - accepts(ref) up to the merge point, states[j][i] =
// own state at the end of chunk j for chunks before the merge.
template <int MODE>
__global__ void __launch_bounds__(1024) k_fuse_ref(DevImage img, const uint8_t* __restrict__ in, uint64_t len,
                                                   uint32_t B, const uint32_t* __restrict__ cand,
                                                   const uint32_t* __restrict__ ncand_p, uint32_t max_chunks,
                                                   uint32_t* __restrict__ states, uint32_t* __restrict__ merged,
                                                   long long* __restrict__ dcnt, uint32_t* __restrict__ unmerged) {
  extern __shared__ __align__(1024) uint8_t smem[];
  stage_table(img, smem);
  __syncthreads();
  using S = Step<MODE>;
  const uint32_t ncand = *ncand_p;
  uint32_t um = 0;
  for (uint32_t i = threadIdx.x; i < ncand; i += blockDim.x) {
    uint32_t code = __ldg(img.tid2code + cand[i]), rcode = __ldg(img.tid2code + cand[0]);
    long long d = 0;
    uint32_t mj = code == rcode ? 0 : kNoState;
    const uint64_t N = (len + B - 1) / B;
    for (uint32_t j = 0; mj == kNoState && j < max_chunks && j < N; j++) {
      const uint64_t lo = (uint64_t)j * B, n = min((uint64_t)B, len - lo);
      const uint8_t* p = in + lo;
      uint64_t t = 0;
      while (t < n) {
        const uint64_t m = min((uint64_t)16, n - t);
        uint32_t a = 0, ra = 0;
        for (uint64_t q = 0; q < m; q++) {
          const uint32_t b = __ldg(p + t + q);
          code = S::byte(img, smem, code, b);
          a += S::acc(code);
          rcode = S::byte(img, smem, rcode, b);
          ra += S::acc(rcode);
        }
        d += (long long)a - (long long)ra;
        t += m;
        if (code == rcode) { mj = j; break; }
      }
      if (mj == kNoState) states[(uint64_t)j * ncand + i] = S::tid(img, code);
    }
    merged[i] = mj;
    dcnt[i] = d;
    um += mj == kNoState;
  }
  if (um) atomicAdd(unmerged, um);
}

// map[cand[i]] = (final of the cand[0] pipeline, its count + dcnt[i]); the pipeline's
// final state and count are read from its control block on the device
// Speculative use (unmerged != null): the pipeline ran before the host knew whether
// every candidate merged; if some did not, every candidate's entry becomes kInvalidMap
// and the composition on every rank reports it (all ranks then redo the exact map).
__global__ void k_map_fused(const uint32_t* __restrict__ cand, const uint32_t* __restrict__ ncand_p,
                            const long long* __restrict__ dcnt, const uint32_t* __restrict__ fin_p,
                            const unsigned long long* __restrict__ count_p, uint32_t* __restrict__ mend,
                            unsigned long long* __restrict__ mcnt, const uint32_t* __restrict__ unmerged) {
  const uint32_t ncand = *ncand_p;
  const uint32_t fin = (unmerged && *unmerged) ? kInvalidMap : *fin_p;
  const unsigned long long c0 = *count_p;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < ncand; i += gridDim.x * blockDim.x) {
    mend[cand[i]] = fin;
    mcnt[cand[i]] = (unsigned long long)((long long)c0 + dcnt[i]);
  }
}

// P2P exchange (p2p.cu), fused mode: ONE kernel computes this rank's map entries (as
// k_map_fused) and sends the finished map to every peer — one CTA writes the candidates'
// entries, then stores the whole map (k_map_init wrote the rest earlier in the stream) into
// slot [rank] of every peer's mailbox, fences system-wide and raises its flag there.
__global__ void __launch_bounds__(1024) k_map_fused_publish(
    const uint32_t* __restrict__ cand, const uint32_t* __restrict__ ncand_p, const long long* __restrict__ dcnt,
    const uint32_t* __restrict__ fin_p, const unsigned long long* __restrict__ count_p, uint32_t* __restrict__ mend,
    unsigned long long* __restrict__ mcnt, const uint32_t* __restrict__ unmerged, uint64_t mapb,
    uint8_t* const* __restrict__ peers, uint32_t G, uint32_t rank, uint32_t set, unsigned long long seq) {
  const uint32_t ncand = *ncand_p;
  const uint32_t fin = (unmerged && *unmerged) ? kInvalidMap : *fin_p;
  const unsigned long long c0 = *count_p;
  for (uint32_t i = threadIdx.x; i < ncand; i += blockDim.x) {
    mend[cand[i]] = fin;
    mcnt[cand[i]] = (unsigned long long)((long long)c0 + dcnt[i]);
  }
  __syncthreads();  // the whole map is final (block-scope: this CTA wrote the candidates)
  __threadfence();
  const uint4* src = reinterpret_cast<const uint4*>(mend);
  const uint64_t words = mapb / 16;
  for (uint32_t g = 0; g < G; g++) {
    if (g == rank) continue;
    uint4* dst = reinterpret_cast<uint4*>(peers[g] + ((uint64_t)set * G + rank) * mapb);
    for (uint64_t i = threadIdx.x; i < words; i += blockDim.x) dst[i] = __ldcg(src + i);
  }
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x < G && threadIdx.x != rank) {
    unsigned long long* flags = reinterpret_cast<unsigned long long*>(peers[threadIdx.x] + 2ull * G * mapb);
    *reinterpret_cast<volatile unsigned long long*>(flags + (uint64_t)set * G + rank) = seq;
  }
}

// finish (fused mode): locate this rank's start among the candidates and write
// the chunk ends walked before it merged with the reference path
__global__ void k_fix_prefix_fused(const uint32_t* __restrict__ states, const uint32_t* __restrict__ cand,
                                   const uint32_t* __restrict__ ncand_p, const uint32_t* __restrict__ merged,
                                   const uint32_t* __restrict__ srank_p, const uint32_t* __restrict__ inv,
                                   uint32_t poison, uint32_t* __restrict__ chunk_ends, uint32_t* __restrict__ err) {
  __shared__ uint32_t ci;
  if (srank_p[2] != 0) return;  // the composition failed (e.g. an invalid speculative map): nothing to fix
  const uint32_t ncand = *ncand_p, sr = *srank_p;
  if (sr == poison) return;  // an invalid byte before this shard: the run reports FSM_ESYMBOL
  if (threadIdx.x == 0) ci = kNoState;
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < ncand; i += blockDim.x)
    if (cand[i] == sr) atomicMin(&ci, i);
  __syncthreads();
  if (ci == kNoState) {
    if (threadIdx.x == 0) *err = 1;
    return;
  }
  const uint32_t nj = merged[ci];
  if (nj == kNoState) {  // this candidate never merged (cannot happen with a valid map)
    if (threadIdx.x == 0) *err = 1;
    return;
  }
  for (uint32_t j = threadIdx.x; j < nj; j += blockDim.x) chunk_ends[j] = inv[states[(uint64_t)j * ncand + ci]];
}

__global__ void k_set_u32(uint32_t* p, uint32_t v, uint32_t* p2, uint32_t v2) {
  *p = v;
  if (p2) *p2 = v2;
}

// every entry "not a candidate", except the poison state (transformed id nt - 1), which
// is absorbing and non-accepting (R4): poison -> poison with count 0 on every shard, so
// an invalid byte in an earlier shard composes to the poison final state (FSM_ESYMBOL)
__global__ void k_map_init(uint32_t* __restrict__ mend, unsigned long long* __restrict__ mcnt, uint32_t nt) {
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < nt; s += gridDim.x * blockDim.x) {
    mend[s] = s == nt - 1 ? s : kNoState;
    mcnt[s] = 0;
  }
}

// the map of a rank whose fsm_shard_map failed: the exchange still runs (every rank
// reaches the collective) and every rank's composition reports the failure
__global__ void k_map_error(uint32_t* __restrict__ mend, unsigned long long* __restrict__ mcnt, uint32_t nt,
                            uint32_t code) {
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < nt; s += gridDim.x * blockDim.x) {
    mend[s] = kErrorMap;
    mcnt[s] = s == 0 ? code : 0ull;
  }
}

// map[cand[i]] = (final of its fused path, prefix count + path count)
__global__ void k_map_write(const uint32_t* __restrict__ cand, uint32_t ncand, const uint32_t* __restrict__ grp,
                            const unsigned long long* __restrict__ prefix, const uint32_t* __restrict__ pfinal,
                            const unsigned long long* __restrict__ pcount, uint32_t* __restrict__ mend,
                            unsigned long long* __restrict__ mcnt) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < ncand; i += gridDim.x * blockDim.x) {
    const uint32_t g = grp[i];
    mend[cand[i]] = pfinal[g];
    mcnt[cand[i]] = (prefix ? prefix[i] : 0ull) + pcount[g];
  }
}

// ENUM shard: the whole-shard map for every state.
__global__ void k_map_enum(const uint8_t* __restrict__ topM, const unsigned long long* __restrict__ topC, uint32_t nt,
                           uint32_t* __restrict__ mend, unsigned long long* __restrict__ mcnt) {
  const uint32_t s = threadIdx.x;
  if (s < nt) { mend[s] = topM[s]; mcnt[s] = topC[s]; }
}

// s_0 = q0; s_{h+1} = M_h[s_h]: out = {s_rank, final, err, count_lo, count_hi}.  With
// `staged` the G maps are first copied into shared memory by the whole block (coalesced),
// so the dependent chain of G lookups runs on shared memory instead of G L2 round trips.
// wflags (P2P exchange, p2p.cu; nullptr otherwise): the receiver side of the peer-memory
// exchange fused in — thread 0 first waits (nanosleep spin, bounded ~10 s) until every
// peer's arrival flag of this step equals seq, reports 0 / 1 + the missing rank to
// *wstatus, and only then is any map read (the maps arrive by the peers' remote stores).
__global__ void k_compose(const uint8_t* __restrict__ maps_g, uint32_t G, uint64_t map_bytes, uint64_t cnt_off,
                          uint32_t q0t, uint32_t rank, uint32_t* __restrict__ out, uint32_t staged,
                          const unsigned long long* wflags, unsigned long long seq, uint32_t* wstatus) {
  extern __shared__ __align__(16) uint8_t sm_maps[];
  const uint8_t* maps = maps_g;
  if (wflags) {
    if (threadIdx.x == 0) {
      uint64_t t0, t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
      uint32_t st = 0;
      for (uint32_t g = 0; g < G && !st; g++) {
        if (g == rank) continue;
        while (*reinterpret_cast<const volatile unsigned long long*>(wflags + g) != seq) {
          __nanosleep(200);
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
          if (t - t0 > 20ull * 1000 * 1000 * 1000) {
            st = 1 + g;  // a peer never published this step
            break;
          }
        }
      }
      __threadfence();
      *wstatus = st;
    }
    __syncthreads();
  }
  if (staged) {
    const uint64_t words = G * map_bytes / 4;
    for (uint64_t i = threadIdx.x; i < words; i += blockDim.x)
      reinterpret_cast<uint32_t*>(sm_maps)[i] = __ldcg(reinterpret_cast<const uint32_t*>(maps_g) + i);
    __syncthreads();
    maps = sm_maps;
  }
  if (threadIdx.x || blockIdx.x) return;
  uint32_t s = q0t, srank = q0t, err = 0;
  unsigned long long c = 0;
  for (uint32_t h = 0; h < G; h++) {
    if (h == rank) srank = s;
    const uint32_t* me = reinterpret_cast<const uint32_t*>(maps + h * map_bytes);
    const unsigned long long* mc = reinterpret_cast<const unsigned long long*>(maps + h * map_bytes + cnt_off);
    const uint32_t e = staged ? me[s] : __ldcg(me + s);
    if (e == kErrorMap) {  // rank h's fsm_shard_map failed: report its status and rank
      out[0] = q0t;
      out[1] = q0t;
      out[2] = 3;
      out[3] = (uint32_t)(staged ? mc[0] : __ldcg(mc));
      out[4] = h;
      return;
    }
    if (e == kNoState) { err = 1; break; }
    if (e == kInvalidMap) { err = 2; break; }  // a rank's speculative map must be redone
    c += staged ? mc[s] : __ldcg(mc + s);
    s = e;
  }
  out[0] = srank;
  out[1] = s;
  out[2] = err;
  out[3] = (uint32_t)(c & 0xFFFFFFFFu);
  out[4] = (uint32_t)(c >> 32);
}

// chunk ends [0, nj) of the fused-path prefix of candidate ci
__global__ void k_fix_prefix(const uint32_t* __restrict__ states, uint32_t ncand, uint32_t ci, uint32_t nj,
                             const uint32_t* __restrict__ inv, uint32_t* __restrict__ chunk_ends) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < nj; j += gridDim.x * blockDim.x)
    chunk_ends[j] = inv[states[(uint64_t)j * ncand + ci]];
}

template <int MODE>
cudaError_t fuse_m(const DevImage& img, const uint8_t* in, uint64_t len, uint32_t B, const uint32_t* cand,
                   uint32_t ncand, uint32_t max_chunks, uint32_t* states, unsigned long long* cnt, uint32_t* info,
                   cudaStream_t st) {
  auto kern = k_fuse<MODE>;
  const uint32_t smem = smem_bytes_for(img);
  cudaError_t e = kernel_setup((const void*)kern, smem, 1024, nullptr);
  if (e != cudaSuccess) return e;
  const uint32_t th = ((ncand + 31) / 32) * 32;
  kern<<<1, th, smem, st>>>(img, in, len, B, cand, ncand, max_chunks, states, cnt, info);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_shard_image(const DevImage& img, const uint32_t* ttc, const uint8_t* w, uint32_t L, uint32_t* mark,
                               uint32_t* list, uint32_t* count, cudaStream_t st) {
  k_image<<<1, 1024, 0, st>>>(img, ttc, w, L, mark, list, count);
  return cudaGetLastError();
}

cudaError_t launch_shard_fuse(const DevImage& img, const uint8_t* in, uint64_t len, uint32_t B, const uint32_t* cand,
                              uint32_t ncand, uint32_t max_chunks, uint32_t* states, unsigned long long* cnt,
                              uint32_t* info, cudaStream_t st) {
  switch (img.mode) {
    case MODE_U8: return fuse_m<MODE_U8>(img, in, len, B, cand, ncand, max_chunks, states, cnt, info, st);
    case MODE_U16: return fuse_m<MODE_U16>(img, in, len, B, cand, ncand, max_chunks, states, cnt, info, st);
    case MODE_U16H: return fuse_m<MODE_U16H>(img, in, len, B, cand, ncand, max_chunks, states, cnt, info, st);
    case MODE_U16D: return fuse_m<MODE_U16D>(img, in, len, B, cand, ncand, max_chunks, states, cnt, info, st);
    default: return fuse_m<MODE_U32>(img, in, len, B, cand, ncand, max_chunks, states, cnt, info, st);
  }
}

cudaError_t launch_shard_fuse_ref(const DevImage& img, const uint8_t* in, uint64_t len, uint32_t B,
                                  const uint32_t* cand, const uint32_t* ncand_p, uint32_t max_chunks, uint32_t* states,
                                  uint32_t* merged, long long* dcnt, uint32_t* unmerged, cudaStream_t st) {
  const uint32_t smem = smem_bytes_for(img);
  cudaError_t e;
#define GS_FUSE_REF(M)                                                                                        \
  if ((e = kernel_setup((const void*)k_fuse_ref<M>, smem, 1024, nullptr))) return e;                          \
  k_fuse_ref<M><<<1, 1024, smem, st>>>(img, in, len, B, cand, ncand_p, max_chunks, states, merged, dcnt, unmerged)
  switch (img.mode) {
    case MODE_U8: GS_FUSE_REF(MODE_U8); break;
    case MODE_U16: GS_FUSE_REF(MODE_U16); break;
    case MODE_U16H: GS_FUSE_REF(MODE_U16H); break;
    case MODE_U16D: GS_FUSE_REF(MODE_U16D); break;
    default: GS_FUSE_REF(MODE_U32); break;
  }
#undef GS_FUSE_REF
  return cudaGetLastError();
}

cudaError_t launch_map_fused(const uint32_t* cand, const uint32_t* ncand_p, const long long* dcnt, const uint32_t* fin_p,
                             const unsigned long long* count_p, uint32_t* mend, unsigned long long* mcnt,
                             const uint32_t* unmerged, cudaStream_t st) {
  k_map_fused<<<8, 256, 0, st>>>(cand, ncand_p, dcnt, fin_p, count_p, mend, mcnt, unmerged);
  return cudaGetLastError();
}

cudaError_t launch_map_fused_publish(const uint32_t* cand, const uint32_t* ncand_p, const long long* dcnt,
                                     const uint32_t* fin_p, const unsigned long long* count_p, uint32_t* mend,
                                     unsigned long long* mcnt, const uint32_t* unmerged, uint64_t mapb,
                                     uint8_t* const* peers, uint32_t G, uint32_t rank, uint32_t set,
                                     unsigned long long seq, cudaStream_t st) {
  k_map_fused_publish<<<1, 1024, 0, st>>>(cand, ncand_p, dcnt, fin_p, count_p, mend, mcnt, unmerged, mapb, peers, G,
                                          rank, set, seq);
  return cudaGetLastError();
}

cudaError_t launch_fix_prefix_fused(const uint32_t* states, const uint32_t* cand, const uint32_t* ncand_p,
                                    const uint32_t* merged, const uint32_t* srank_p, const uint32_t* inv,
                                    uint32_t poison, uint32_t* chunk_ends, uint32_t* err, cudaStream_t st) {
  k_fix_prefix_fused<<<1, 256, 0, st>>>(states, cand, ncand_p, merged, srank_p, inv, poison, chunk_ends, err);
  return cudaGetLastError();
}

cudaError_t launch_set_u32(uint32_t* p, uint32_t v, uint32_t* p2, uint32_t v2, cudaStream_t st) {
  k_set_u32<<<1, 1, 0, st>>>(p, v, p2, v2);
  return cudaGetLastError();
}

cudaError_t launch_map_init(uint32_t* mend, unsigned long long* mcnt, uint32_t nt, cudaStream_t st) {
  k_map_init<<<(nt + 255) / 256, 256, 0, st>>>(mend, mcnt, nt);
  return cudaGetLastError();
}

cudaError_t launch_map_error(uint32_t* mend, unsigned long long* mcnt, uint32_t nt, uint32_t code, cudaStream_t st) {
  k_map_error<<<(nt + 255) / 256, 256, 0, st>>>(mend, mcnt, nt, code);
  return cudaGetLastError();
}

cudaError_t launch_map_write(const uint32_t* cand, uint32_t ncand, const uint32_t* grp,
                             const unsigned long long* prefix, const uint32_t* pfinal, const unsigned long long* pcount,
                             uint32_t* mend, unsigned long long* mcnt, cudaStream_t st) {
  k_map_write<<<(ncand + 255) / 256, 256, 0, st>>>(cand, ncand, grp, prefix, pfinal, pcount, mend, mcnt);
  return cudaGetLastError();
}

cudaError_t launch_map_enum(const uint8_t* topM, const unsigned long long* topC, uint32_t nt, uint32_t* mend,
                            unsigned long long* mcnt, cudaStream_t st) {
  k_map_enum<<<1, 64, 0, st>>>(topM, topC, nt, mend, mcnt);
  return cudaGetLastError();
}

cudaError_t launch_compose(const uint8_t* maps, uint32_t G, uint64_t map_bytes, uint64_t cnt_off, uint32_t q0t,
                           uint32_t rank, uint32_t* out, cudaStream_t st, const unsigned long long* wflags,
                           unsigned long long seq, uint32_t* wstatus) {
  const uint64_t bytes = (uint64_t)G * map_bytes;
  uint32_t staged = bytes <= 96 * 1024 && map_bytes % 8 == 0;
  if (staged && kernel_setup((const void*)k_compose, (uint32_t)bytes, 256, nullptr) != cudaSuccess) staged = 0;
  if (staged)
    k_compose<<<1, 256, (uint32_t)bytes, st>>>(maps, G, map_bytes, cnt_off, q0t, rank, out, 1u, wflags, seq, wstatus);
  else
    k_compose<<<1, 32, 0, st>>>(maps, G, map_bytes, cnt_off, q0t, rank, out, 0u, wflags, seq, wstatus);
  return cudaGetLastError();
}

cudaError_t launch_fix_prefix(const uint32_t* states, uint32_t ncand, uint32_t ci, uint32_t nj, const uint32_t* inv,
                              uint32_t* chunk_ends, cudaStream_t st) {
  if (!nj) return cudaSuccess;
  k_fix_prefix<<<(nj + 255) / 256, 256, 0, st>>>(states, ncand, ci, nj, inv, chunk_ends);
  return cudaGetLastError();
}

}  // namespace gspec
