// literal.cu — SURVEY §8(f) f4: the paper-literal single-CTA kernel.
//
// Alg. 2 L2-6 for round 0, then Alg. 3 SPEC_RECOVERY_END
// exactly as printed: one thread per chunk (T = N <= 1024, one CTA), a shared
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

template <int MODE>
__global__ void __launch_bounds__(kLitMax) k_literal_sre(DevImage img, RunParams rp, RecStore rs, Ctl* ctl,
                                                        uint32_t* __restrict__ chunk_ends) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t endc_sh[kLitMax];
  __shared__ int mark;
  __shared__ unsigned long long red[kLitMax / 32][4];
  using S = Step<MODE>;
  stage_table(img, smem);
  const uint32_t N = (uint32_t)rp.N, c = threadIdx.x, cap = rp.vr_end;
  const bool act = c < N;
  const uint64_t lo = (uint64_t)c * rp.B, n = act ? min((uint64_t)rp.B, rp.len - lo) : 0;
  const uint8_t* p = rp.in + lo;
  if (act) rs.n_end[c] = 0;
  __syncthreads();
  auto run = [&](uint32_t st, uint32_t* cnt) {  // FSM_Processing(fsm, Pi(c), st)
    uint32_t acc = 0;
    const uint32_t code = walk_bytes<MODE>(img, smem, p, n, __ldg(img.tid2code + st), acc);
    *cnt = acc;
    return S::tid(img, code);
  };
  // Alg. 2 L3-6: predict (lookback-2 over the previous chunk's last bytes), run QS.front()
  uint32_t endc = 0;
  unsigned long long checks = 0, matches = 0, tasks = 0, reread = 0;
  if (act) {
    const uint32_t st = c == 0 ? rp.q0t : __ldg(img.qs2 + (uint64_t)qs_pair(img, rp.in, c, rp.B) * kQsMax);
    uint32_t cnt;
    endc = run(st, &cnt);
    lit_push(rs, cap, c, st, endc, cnt);
  }
  uint32_t rounds = 0;
  // Alg. 3 L4-18
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
    if (c == f) mark = found;  // L12-13
    f++;                       // L14
    __syncthreads();           // L15
    if (!mark) {               // L16-18
      rounds++;
      if (act && !found) {
        uint32_t cnt;
        endc = run(endp, &cnt);
        lit_push(rs, cap, c, endp, endc, cnt);
        tasks++;
        reread += n;
      }
    }
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
  unsigned long long v[4] = {total, checks, matches, tasks};
#pragma unroll
  for (int k = 0; k < 4; k++)
    for (int o = 16; o > 0; o >>= 1) v[k] += __shfl_down_sync(0xffffffffu, v[k], o);
  if ((c & 31) == 0)
    for (int k = 0; k < 4; k++) red[c >> 5][k] = v[k];
  unsigned long long rr = reread;
  for (int o = 16; o > 0; o >>= 1) rr += __shfl_down_sync(0xffffffffu, rr, o);
  __syncthreads();
  if (c == 0) {
    unsigned long long s[4] = {0, 0, 0, 0};
    for (uint32_t w = 0; w < blockDim.x / 32; w++)
      for (int k = 0; k < 4; k++) s[k] += red[w][k];
    ctl->accept_count = s[0];
    ctl->verify_checks = s[1];
    ctl->verify_matches = s[2];
    ctl->rounds = rounds;
    ctl->tasks_mustdo = rounds;
    ctl->tasks_sre = s[3] - rounds;
    ctl->active_sum = s[3];
    ctl->xfin = endc_sh[N - 1];
  }
  __syncthreads();
  if ((c & 31) == 0) atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->reread_bytes), rr);
}

template <int MODE>
cudaError_t launch_lit(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* ctl, uint32_t* ce,
                       cudaStream_t st) {
  auto kern = k_literal_sre<MODE>;
  const uint32_t smem = smem_bytes_for(img);
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
