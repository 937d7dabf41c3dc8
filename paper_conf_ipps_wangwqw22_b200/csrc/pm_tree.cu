// pm_tree.cu — SURVEY §8(f) f2: a faithful replica of PM (Parallel Merge, Xia et al.,
// the paper's prior state of the art: Fig. 2; cost model Eq. 2).
//
//   round 0   spec-k speculative execution (the TMA spec kernel with k paths):
//             chunk c's records (s_j, e_j, cnt_j), j < k.
//   stage 1   "parallel tree-like verification": ceil(log2 N) merge rounds.  Level l
//             holds, for each segment [g 2^l, (g+1) 2^l), a k-entry map keyed by the
//             starts of its first chunk.  A merge looks a valid left entry's end up
//             among the right segment's starts; a miss marks the path INVALID instead
//             of re-executing anything ("delayed recovery").  One thread per
//             output segment, one launch per level.
//   stage 2   "sequential verification and recovery" (Eq. 2's second sum): one thread
//             walks from q0 over the merged segments, taking the largest segment that
//             starts at the current chunk and holds a valid entry for the current state;
//             a state that is not among the chunk's speculated starts is recovered at
//             once by walking that chunk (the must-be-done recovery).  Its decisions go
//             to a jump list.
//   descent   one thread per chunk finds its jump (binary search), descends the merges
//             (left child: same entry, right child: the entry the left end matched) and
//             writes the chunk's end state.
// Tests compare results and every stage counter with a CPU simulation of the same steps.
#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr uint32_t kNo = 0xFFFFFFFFu;
constexpr uint32_t kValid = 0x80000000u;

struct PmEnt {
  uint32_t end;
  uint32_t flags;  // kValid | right-child entry index (merge levels)
  unsigned long long cnt;
};

__device__ __forceinline__ void block_add(unsigned long long v, unsigned long long* dst) {
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
}

// level 0 = the round-0 records; starts[c][j] (kNo where the chunk has fewer than k)
__global__ void k_pm_level0(RecStore rs, uint64_t N, uint32_t k, PmEnt* __restrict__ lv0,
                            uint32_t* __restrict__ starts) {
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < N; c += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t ne = min(__ldcg(rs.n_end + c), k);
    for (uint32_t j = 0; j < k; j++) {
      PmEnt e{0u, 0u, 0ull};
      uint32_t s = kNo;
      if (j < ne) {
        s = __ldcg(rs.start + (uint64_t)j * rs.cap + c);
        e.end = __ldcg(rs.end + (uint64_t)j * rs.cap + c);
        e.cnt = __ldcg(rs.cnt + (uint64_t)j * rs.cap + c);
        e.flags = kValid;
      }
      lv0[c * k + j] = e;
      starts[c * k + j] = s;
    }
  }
}

// one merge round: segments of level l from pairs of level l-1
__global__ void k_pm_merge(const PmEnt* __restrict__ prev, uint64_t nprev, PmEnt* __restrict__ out, uint64_t nseg,
                           uint32_t l, uint32_t k, const uint32_t* __restrict__ starts,
                           unsigned long long* __restrict__ stats) {
  unsigned long long checks = 0, invalid = 0;
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < nseg; g += (uint64_t)gridDim.x * blockDim.x) {
    const PmEnt* le = prev + 2 * g * k;
    PmEnt* o = out + g * k;
    if (2 * g + 1 >= nprev) {  // unpaired last segment: moves up unchanged
      for (uint32_t j = 0; j < k; j++) o[j] = le[j];
      continue;
    }
    const PmEnt* re = prev + (2 * g + 1) * k;
    const uint64_t m1 = (2 * g + 1) << (l - 1);  // first chunk of the right segment
    uint32_t rs_[kQsMax];
    for (uint32_t r = 0; r < k; r++) rs_[r] = starts[m1 * k + r];
    for (uint32_t j = 0; j < k; j++) {
      const PmEnt a = le[j];
      PmEnt res{0u, 0u, 0ull};
      if (a.flags & kValid) {
        checks++;
        uint32_t hit = kNo;
        for (uint32_t r = 0; r < k; r++)
          if (hit == kNo && rs_[r] == a.end) hit = r;
        if (hit != kNo && (re[hit].flags & kValid)) {
          res.end = re[hit].end;
          res.cnt = a.cnt + re[hit].cnt;
          res.flags = kValid | hit;
        } else {
          invalid++;  // delayed recovery: the path is marked, not re-executed
        }
      }
      o[j] = res;
    }
  }
  block_add(checks, stats + 0);
  block_add(invalid, stats + 1);
}

// stage 2 (one thread; the table is staged for its recovery walks).  Jump list entry:
// {first chunk, level (kNo = recovery), entry j (recovery: its start state)}.
template <int MODE>
__global__ void k_pm_stage2(DevImage img, RunParams rp, const PmEnt* __restrict__ lv, const uint64_t* __restrict__ lvoff,
                            uint32_t L, uint32_t k, const uint32_t* __restrict__ starts, uint32_t* __restrict__ jl,
                            uint32_t* __restrict__ rec_end, Ctl* ctl, unsigned long long* __restrict__ stats) {
  extern __shared__ __align__(1024) uint8_t smem[];
  using S = Step<MODE>;
  stage_table(img, smem);
  __syncthreads();
  if (threadIdx.x != 0) return;
  const uint64_t N = rp.N;
  uint32_t t = rp.q0t;
  uint64_t c = 0, njump = 0, recov = 0, checks = 0, reread = 0;
  unsigned long long total = 0;
  while (c < N) {
    uint32_t jf = kNo;
    for (uint32_t j = 0; j < k; j++)
      if (jf == kNo && starts[c * k + j] == t) jf = j;
    checks++;
    bool done = false;
    if (jf != kNo) {
      uint32_t lmax = 0;
      while (lmax < L && (c & ((2ull << lmax) - 1)) == 0) lmax++;
      for (int l = (int)lmax; l >= 0 && !done; l--) {
        const PmEnt e = lv[lvoff[l] + (c >> l) * k + jf];
        if (!(e.flags & kValid)) continue;
        jl[3 * njump] = (uint32_t)c;
        jl[3 * njump + 1] = (uint32_t)l;
        jl[3 * njump + 2] = jf;
        njump++;
        total += e.cnt;
        t = e.end;
        c = min(N, ((c >> l) + 1) << l);
        done = true;
      }
    }
    if (!done) {  // must-be-done recovery of chunk c (Eq. 2: T_comm(1) + T_ver(k) + T_p1)
      const uint64_t lo = c * rp.B, n = min((uint64_t)rp.B, rp.len - lo);
      uint32_t acc = 0;
      const uint32_t code = walk_bytes<MODE>(img, smem, rp.in + lo, n, __ldg(img.tid2code + t), acc);
      jl[3 * njump] = (uint32_t)c;
      jl[3 * njump + 1] = kNo;
      jl[3 * njump + 2] = t;
      njump++;
      t = S::tid(img, code);
      rec_end[c] = t;
      total += acc;
      recov++;
      reread += n;
      c++;
    }
  }
  ctl->xfin = t;
  ctl->accept_count = total;
  ctl->rounds = L;
  ctl->tasks_mustdo = recov;
  ctl->active_sum = recov;
  ctl->reread_bytes = reread;
  ctl->verify_checks = checks;
  ctl->verify_matches = njump - recov;
  ctl->ntask[0] = njump;
  ctl->pm_merge_checks = stats[0];
  ctl->pm_invalid_marks = stats[1];
  ctl->pm_jumps = njump - recov;
}

// per chunk: its jump-list entry, then down the merges to the chunk's own entry
__global__ void k_pm_descent(const PmEnt* __restrict__ lv, const uint64_t* __restrict__ lvoff, uint32_t k,
                             const uint32_t* __restrict__ jl, const Ctl* __restrict__ ctl,
                             const uint32_t* __restrict__ rec_end, const uint32_t* __restrict__ inv, uint64_t N,
                             uint32_t* __restrict__ chunk_ends) {
  const uint64_t nj = ctl->ntask[0];
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < N; c += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t a = 0, z = nj - 1;  // last entry whose first chunk <= c
    while (a < z) {
      const uint64_t mid = (a + z + 1) / 2;
      if (jl[3 * mid] <= c) a = mid; else z = mid - 1;
    }
    const uint32_t l0 = jl[3 * a + 1];
    uint32_t e;
    if (l0 == kNo) {
      e = rec_end[c];
    } else {
      uint32_t j = jl[3 * a + 2];
      for (uint32_t l = l0; l > 0; l--) {
        const uint64_t g = c >> l, child = c >> (l - 1);
        if (child & 1) j = lv[lvoff[l] + g * k + j].flags & ~kValid;  // right child: the matched entry
      }
      e = lv[c * k + j].end;
    }
    chunk_ends[c] = __ldg(inv + e);
  }
}

template <int MODE>
cudaError_t stage2_m(const DevImage& img, const RunParams& rp, const void* lv, const uint64_t* lvoff, uint32_t L,
                     uint32_t k, const uint32_t* starts, uint32_t* jl, uint32_t* rec_end, Ctl* ctl,
                     unsigned long long* stats, cudaStream_t st) {
  auto kern = k_pm_stage2<MODE>;
  const uint32_t smem = smem_bytes_for(img);
  cudaError_t e = kernel_setup((const void*)kern, smem, 128, nullptr);
  if (e != cudaSuccess) return e;
  kern<<<1, 128, smem, st>>>(img, rp, reinterpret_cast<const PmEnt*>(lv), lvoff, L, k, starts, jl, rec_end, ctl,
                             stats);
  return cudaGetLastError();
}

}  // namespace

uint64_t pm_tree_scratch_bytes(uint64_t N, uint32_t k, uint32_t* levels) {
  uint32_t L = 0;
  while ((1ull << L) < N) L++;
  uint64_t ents = 0;
  for (uint32_t l = 0; l <= L; l++) ents += ((N + (1ull << l) - 1) >> l) * k;
  if (levels) *levels = L;
  // entries + starts + jump list (3 u32 per chunk) + recovery ends + level offsets + stats
  return ents * sizeof(PmEnt) + N * k * 4 + N * 12 + N * 4 + 64 * 8 + 64 + 1024;
}

// Stream-ordered PM-tree verification after the spec-k kernel (records in rs).
cudaError_t launch_pm_tree(const DevImage& img, const RunParams& rp, const RecStore& rs, uint32_t k, void* scratch,
                           Ctl* ctl, uint32_t* d_chunk_ends, int sms, cudaStream_t st, uint32_t* launches) {
  const uint64_t N = rp.N;
  uint32_t L = 0;
  pm_tree_scratch_bytes(N, k, &L);
  uint64_t off[64];
  uint64_t ents = 0;
  for (uint32_t l = 0; l <= L; l++) {
    off[l] = ents;
    ents += ((N + (1ull << l) - 1) >> l) * k;
  }
  uint8_t* p = static_cast<uint8_t*>(scratch);
  PmEnt* lv = reinterpret_cast<PmEnt*>(p);
  p += ents * sizeof(PmEnt);
  uint32_t* starts = reinterpret_cast<uint32_t*>(p);
  p += N * k * 4;
  uint32_t* jl = reinterpret_cast<uint32_t*>(p);
  p += N * 12;
  uint32_t* rec_end = reinterpret_cast<uint32_t*>(p);
  p += N * 4;
  uint64_t* d_off = reinterpret_cast<uint64_t*>(p);
  p += 64 * 8;
  unsigned long long* stats = reinterpret_cast<unsigned long long*>(p);
  cudaError_t e;
  if ((e = cudaMemcpyAsync(d_off, off, 8ull * (L + 1), cudaMemcpyHostToDevice, st)) != cudaSuccess) return e;
  if ((e = cudaMemsetAsync(stats, 0, 64, st)) != cudaSuccess) return e;
  const uint32_t grid0 = (uint32_t)std::min<uint64_t>((N + 255) / 256, (uint64_t)sms * 8);
  k_pm_level0<<<grid0, 256, 0, st>>>(rs, N, k, lv, starts);
  uint32_t nl = 1;
  for (uint32_t l = 1; l <= L; l++) {
    const uint64_t nprev = (N + (1ull << (l - 1)) - 1) >> (l - 1), nseg = (N + (1ull << l) - 1) >> l;
    const uint32_t grid = (uint32_t)std::min<uint64_t>((nseg + 127) / 128, (uint64_t)sms * 8);
    k_pm_merge<<<grid, 128, 0, st>>>(lv + off[l - 1], nprev, lv + off[l], nseg, l, k, starts, stats);
    nl++;
  }
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  switch (img.mode) {
    case MODE_U8: e = stage2_m<MODE_U8>(img, rp, lv, d_off, L, k, starts, jl, rec_end, ctl, stats, st); break;
    case MODE_U16: e = stage2_m<MODE_U16>(img, rp, lv, d_off, L, k, starts, jl, rec_end, ctl, stats, st); break;
    case MODE_U16H: e = stage2_m<MODE_U16H>(img, rp, lv, d_off, L, k, starts, jl, rec_end, ctl, stats, st); break;
    case MODE_U16D: e = stage2_m<MODE_U16D>(img, rp, lv, d_off, L, k, starts, jl, rec_end, ctl, stats, st); break;
    default: e = stage2_m<MODE_U32>(img, rp, lv, d_off, L, k, starts, jl, rec_end, ctl, stats, st); break;
  }
  if (e != cudaSuccess) return e;
  nl++;
  if (d_chunk_ends) {
    k_pm_descent<<<grid0, 256, 0, st>>>(lv, d_off, k, jl, ctl, rec_end, img.inv, N, d_chunk_ends);
    nl++;
  }
  *launches = nl;
  return cudaGetLastError();
}

}  // namespace gspec
