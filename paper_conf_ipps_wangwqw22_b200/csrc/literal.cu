// literal.cu — SURVEY §8(f) f4: the paper-literal single-CTA kernels.
//
// Alg. 2 L2-6 for round 0, then Alg. 3 SPEC_RECOVERY_END,
// or its RR / NF variants (Alg. 4, Alg. 5), exactly as printed: one thread per chunk (T = N <= 1024, one CTA), a shared
// `mark`, one frontier step per iteration (`f++`, L14) with a `sync()` (L15),
// exactly N iterations.  It is the reference point for the batched-frontier
// redesign in verify_recover.cu (reading R13): same results, but every
// iteration is a CTA-wide barrier and a must-do recovery is a single-thread walk
// on the critical path.  Tests compare it with a CPU simulation of the same steps.
#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr uint32_t kLitMax = 1024;  // threads = chunks

__device__ __forceinline__ bool lit_lookup(const RecStore& rs, uint32_t cap, uint32_t c, uint32_t x, uint32_t* end,
                                           uint32_t* cnt) {
  const uint32_t n = min(rs.n_end[c], cap);
  for (uint32_t s = 0; s < n; s++)
    if (rs.start[(uint64_t)s * rs.cap + c] == x) {
      *end = rs.end[(uint64_t)s * rs.cap + c];
      if (cnt) *cnt = rs.cnt[(uint64_t)s * rs.cap + c];
      return true;
    }
  return false;
}

__device__ __forceinline__ void lit_push(const RecStore& rs, uint32_t cap, uint32_t c, uint32_t st, uint32_t e,
                                         uint32_t cnt) {
  const uint32_t n = rs.n_end[c];
  const uint64_t o = (uint64_t)(n % cap) * rs.cap + c;  // FIFO ring (reading R16)
  rs.start[o] = st;
  rs.end[o] = e;
  rs.cnt[o] = cnt;
  rs.n_end[c] = n + 1;
}

// Exclusive block scan of one value per thread (threads = chunks, <= 1024).
__device__ __forceinline__ uint32_t lit_excl_scan(uint32_t v, uint32_t* wsum, uint32_t* total) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x / 32;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) wsum[warp] = x;
  __syncthreads();
  if (warp == 0) {
    uint32_t w = lane < nw ? wsum[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= (uint32_t)o) w += y;
    }
    if (lane < nw) wsum[lane] = w;
  }
  __syncthreads();
  const uint32_t ex = x - v + (warp > 0 ? wsum[warp - 1] : 0u);
  *total = wsum[nw - 1];
  __syncthreads();
  return ex;
}

// Alg. 3 (SRE), Alg. 4 (RR), Alg. 5 (NF) as printed: one thread per chunk, N iterations
// of the frontier step (L4-15); when mark == false the recovery step of rp.scheme runs,
// 0-indexed with the frontier chunk fr = f before L14's increment (readings R10, R21):
//   SRE: every thread with found == false re-executes its chunk from endp (L16-18).
//   RR / NF: threads tid >= fr re-execute their own chunk from endp (L19-21 / NF_Sched
//   L26-27; verbatim, even when found); threads tid < fr dequeue a start from another
//   chunk's QS: RR chunk fr+1 + tid mod (N-fr-1) (L23-25), NF the first non-empty QS of
//   chunks fr+1, fr+2, ... (L29-33).  The concurrent queues are resolved in tid
//   order: the r-th thread dequeuing QS_c gets its r-th remaining entry; none left -> idle.
//   QS_c = lookback-2 ranking (qs_cap), dequeues start at entry 1 (round 0 ran the front,
//   R9).  Records are pushed to VR_cid in tid order (helpers, then the chunk's own thread);
//   a thread tid >= fr with found == false takes its new end (L28-29).
__host__ __device__ inline uint32_t lit_arrays_off(const DevImage& img) { return (smem_bytes_for(img) + 15u) & ~15u; }

template <int MODE>
__global__ void __launch_bounds__(kLitMax) k_literal(DevImage img, RunParams rp, RecStore rs, Ctl* ctl,
                                                    uint32_t* __restrict__ chunk_ends) {
  extern __shared__ __align__(1024) uint8_t smem[];
  // the per-chunk arrays live in dynamic shared memory behind the table: the table must start
  // near the shared window's base (a delta-row image holds absolute 16-bit row offsets)
  uint32_t* endc_sh = reinterpret_cast<uint32_t*>(smem + lit_arrays_off(img));
  uint32_t* pair_sh = endc_sh + kLitMax;   // QS_c = qs2[pair_sh[c]] (chunk 0: [q0])
  uint32_t* cur_sh = pair_sh + kLitMax;    // QS_c dequeue cursor
  uint32_t* pre_sh = cur_sh + kLitMax;     // NF: exclusive prefix of the remaining entries
  uint32_t* take_sh = pre_sh + kLitMax;    // entries of QS_c dequeued by helpers this iteration
  __shared__ uint32_t wsum[32];
  __shared__ int mark;
  __shared__ unsigned long long red[kLitMax / 32][6];
  using S = Step<MODE>;
  stage_table(img, smem);
  const int scheme = rp.scheme;
  const uint32_t N = (uint32_t)rp.N, c = threadIdx.x, cap = rp.vr_end;
  const bool act = c < N;
  const uint32_t pair = (act && c > 0) ? qs_pair(img, rp.in, c, rp.B) : 0u;
  const uint32_t ql = (act && c > 0) ? min((uint32_t)__ldg(img.qs2_len + pair), rp.qs_cap) : 1u;
  pair_sh[c] = pair;
  cur_sh[c] = 1;  // R9: round 0 consumed QS.front()
  if (act) rs.n_end[c] = 0;
  __syncthreads();
  auto run = [&](uint32_t cid, uint32_t st, uint32_t* cnt) {  // FSM_Processing(fsm, Pi(cid), st)
    uint32_t acc = 0;
    const uint64_t lo = (uint64_t)cid * rp.B, n = min((uint64_t)rp.B, rp.len - lo);
    const uint32_t code = walk_bytes<MODE>(img, smem, rp.in + lo, n, __ldg(img.tid2code + st), acc);
    *cnt = acc;
    return S::tid(img, code);
  };
  auto qs_at = [&](uint32_t cid, uint32_t j) {  // QS_cid[j]
    return cid == 0 ? rp.q0t : __ldg(img.qs2 + (uint64_t)pair_sh[cid] * kQsMax + j);
  };
  // Alg. 2 L3-6: predict (lookback-2 over the previous chunk's last bytes), run QS.front()
  uint32_t endc = 0;
  unsigned long long checks = 0, matches = 0, n_mustdo = 0, n_sre = 0, n_hel = 0, reread = 0;
  if (act) {
    const uint32_t st = qs_at(c, 0);
    uint32_t cnt;
    endc = run(c, st, &cnt);
    lit_push(rs, cap, c, st, endc, cnt);
  }
  uint32_t rounds = 0;
  // Alg. 3 L4-18 (Alg. 4 / 5 L16-29)
  for (uint32_t f = 0; f < N;) {
    if (act) endc_sh[c] = endc;
    __syncthreads();
    const uint32_t endp = c == 0 ? rp.q0t : endc_sh[act ? c - 1 : 0];  // L6: end_state_comm(endc)
    bool found = false;
    if (act) {  // L7-11
      uint32_t e;
      found = lit_lookup(rs, cap, c, endp, &e, nullptr);
      checks++;
      if (found) {
        matches++;
        endc = e;
      }
    }
    const uint32_t fr = f;
    if (c == f) mark = found;  // L12-13
    f++;                       // L14
    __syncthreads();           // L15
    if (mark) continue;        // L16-17
    rounds++;
    // ---- assignment: (cid, st) per thread, pos = its rank among VR_cid's pushes
    uint32_t cid = 0xFFFFFFFFu, st = 0, pos = 0, take = 0;
    if (scheme == FSM_SCHEME_SRE) {
      if (act && !found) { cid = c; st = endp; }
    } else {
      const uint32_t M = N - fr - 1;
      const uint32_t rem = (act && c > fr) ? (ql > cur_sh[c] ? ql - cur_sh[c] : 0u) : 0u;
      if (scheme == FSM_SCHEME_RR) {
        if (act && c > fr) {  // helpers tid < fr with tid mod M == c - fr - 1
          const uint32_t u = c - fr - 1;
          take = u < fr ? min(rem, (fr - u + M - 1) / M) : 0u;
        }
      } else {  // NF: the first fr entries of QS_{fr+1} || QS_{fr+2} || ...
        uint32_t tot;
        const uint32_t pre = lit_excl_scan(rem, wsum, &tot);
        pre_sh[c] = pre;
        take = fr > pre ? min(rem, fr - pre) : 0u;
      }
      take_sh[c] = take;
      __syncthreads();
      if (act && c >= fr) {  // frontier / rear thread: own chunk from endp, pushed after the helpers
        cid = c;
        st = endp;
        pos = take;
      } else if (act && M > 0) {  // helper
        uint32_t d = 0xFFFFFFFFu, j = 0;
        if (scheme == FSM_SCHEME_RR) {
          const uint32_t t = fr + 1 + c % M, r = c / M;
          if (r < take_sh[t]) { d = t; j = r; }
        } else {
          uint32_t a = fr + 1, z = N - 1;  // last chunk with pre <= c
          while (a < z) {
            const uint32_t mid = (a + z + 1) / 2;
            if (pre_sh[mid] <= c) a = mid; else z = mid - 1;
          }
          if (c - pre_sh[a] < take_sh[a]) { d = a; j = c - pre_sh[a]; }
        }
        if (d != 0xFFFFFFFFu) {
          cid = d;
          st = qs_at(d, cur_sh[d] + j);
          pos = j;
        }
      }
    }
    // ---- execute (pure walks), push to VR_cid in tid order
    uint32_t e2 = 0, cnt2 = 0;
    if (cid != 0xFFFFFFFFu) {
      e2 = run(cid, st, &cnt2);
      reread += min((uint64_t)rp.B, rp.len - (uint64_t)cid * rp.B);
      if (cid != c) n_hel++; else if (c == fr) n_mustdo++; else n_sre++;
    }
    __syncthreads();  // every thread's lookups of this iteration are done: pushes may land
    if (cid != 0xFFFFFFFFu) {
      const uint32_t total = scheme == FSM_SCHEME_SRE ? 1u : take_sh[cid] + 1u;
      if (pos + cap >= total) {  // FIFO: a push that a later push of this iteration evicts is dropped
        const uint64_t o = (uint64_t)((rs.n_end[cid] + pos) % cap) * rs.cap + cid;
        rs.start[o] = st;
        rs.end[o] = e2;
        rs.cnt[o] = cnt2;
      }
    }
    __syncthreads();
    if (act && scheme != FSM_SCHEME_SRE) {
      if (c >= fr) rs.n_end[c] += take_sh[c] + 1;
      if (c > fr) cur_sh[c] += take_sh[c];
    } else if (act && cid == c) {
      rs.n_end[c] += 1;
    }
    if (act && cid == c && !found) endc = e2;  // L17 / L28-29
    __syncthreads();
  }
  // every chunk verified: true start of chunk c = endc of c-1 (q0 for chunk 0)
  if (act) endc_sh[c] = endc;
  __syncthreads();
  unsigned long long total = 0;
  if (act) {
    uint32_t e, cnt = 0;
    lit_lookup(rs, cap, c, c == 0 ? rp.q0t : endc_sh[c - 1], &e, &cnt);
    total = cnt;
    if (chunk_ends) chunk_ends[c] = __ldg(img.inv + endc);
  }
  unsigned long long v[6] = {total, checks, matches, n_sre, n_hel, reread};
#pragma unroll
  for (int k = 0; k < 6; k++)
    for (int o = 16; o > 0; o >>= 1) v[k] += __shfl_down_sync(0xffffffffu, v[k], o);
  if ((c & 31) == 0)
    for (int k = 0; k < 6; k++) red[c >> 5][k] = v[k];
  __syncthreads();
  if (c == 0) {
    unsigned long long s6[6] = {0, 0, 0, 0, 0, 0};
    for (uint32_t w = 0; w < blockDim.x / 32; w++)
      for (int k = 0; k < 6; k++) s6[k] += red[w][k];
    ctl->accept_count = s6[0];
    ctl->verify_checks = s6[1];
    ctl->verify_matches = s6[2];
    ctl->rounds = rounds;
    ctl->tasks_mustdo = rounds;  // the frontier thread re-executes in every round (mark == false)
    ctl->tasks_sre = s6[3];
    ctl->tasks_helper = s6[4];
    ctl->active_sum = rounds + s6[3] + s6[4];
    ctl->reread_bytes = s6[5];
    ctl->xfin = endc_sh[N - 1];
  }
  (void)n_mustdo;
}

template <int MODE>
cudaError_t launch_lit(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* ctl, uint32_t* ce,
                       cudaStream_t st) {
  auto kern = k_literal<MODE>;
  const uint32_t smem = lit_arrays_off(img) + 5 * kLitMax * 4;
  cudaError_t e = kernel_setup((const void*)kern, smem, kLitMax, nullptr);
  if (e != cudaSuccess) return e;
  const uint32_t threads = (uint32_t)((rp.N + 31) / 32 * 32);
  kern<<<1, threads, smem, st>>>(img, rp, rs, ctl, ce);
  return cudaGetLastError();
}

}  // namespace

uint32_t literal_max_chunks() { return kLitMax; }

cudaError_t launch_literal_sre(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* ctl,
                               uint32_t* d_chunk_ends, cudaStream_t st) {
  switch (img.mode) {
    case MODE_U8: return launch_lit<MODE_U8>(img, rp, rs, ctl, d_chunk_ends, st);
    case MODE_U16: return launch_lit<MODE_U16>(img, rp, rs, ctl, d_chunk_ends, st);
    case MODE_U16H: return launch_lit<MODE_U16H>(img, rp, rs, ctl, d_chunk_ends, st);
    case MODE_U16D: return launch_lit<MODE_U16D>(img, rp, rs, ctl, d_chunk_ends, st);
    default: return launch_lit<MODE_U32>(img, rp, rs, ctl, d_chunk_ends, st);
  }
}

}  // namespace gspec
