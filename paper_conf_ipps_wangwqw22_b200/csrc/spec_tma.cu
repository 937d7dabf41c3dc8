// spec_tma.cu — B2 fast path: speculative execution with TMA-staged input.
//
// The stream is viewed as a 2-D tensor [N_full chunks][B bytes].  Each warp
// owns tiles of 32 consecutive chunks (lane = chunk, Alg. 2 L3 "Forall
// thread i") and streams them through shared memory with a per-warp
// multi-stage TMA pipeline: box = 32 rows x 64 B, SWIZZLE_64B so the 32
// lanes' 16-byte reads of their own rows are bank-conflict-free.  Lanes then
// run register-resident transition chains over the staged bytes, the
// transformed table resident in shared memory.  One CTA per SM.
#include <cuda.h>

#include <algorithm>
#include <cmath>

#include "internal.h"
#include "walk.cuh"

namespace gspec {
namespace {

constexpr uint32_t kRowBytes = 64;              // box inner extent (bytes per chunk per stage)
constexpr uint32_t kStageBytes = 32 * kRowBytes;  // 32 rows (chunks) per box
constexpr uint32_t kNoTask = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  const uint32_t a = smem_u32(bar);
  while (!done) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  }
}

// The input is streamed exactly once: load it with an L2 evict-first policy so
// it does not push the cold rows of a large transition table out of L2.
__device__ __forceinline__ uint64_t evict_first_policy() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}

__device__ __forceinline__ uint64_t evict_normal_policy() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}

__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar, int32_t x, int32_t y,
                                            uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%2, %3}], [%4], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}

// Blackwell TMA gather: 4 arbitrary rows (chunks) x one 64 B box column.  With
// SWIZZLE_64B the rows land with the same address-based XOR pattern as a 32-row
// 2-D box (tools/gather4_probe.cu verified this at 256 B destination offsets), so
// 8 gathers fill a stage exactly like one tile box and the readers are unchanged.
__device__ __forceinline__ void tma_gather4(void* dst, const CUtensorMap* map, uint64_t* bar, int32_t x, uint4 r,
                                            uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w), "r"(smem_u32(bar)),
      "l"(policy)
      : "memory");
}

// Fused round-0 verification (SRE with spec-1 records, accurate speculation; RunParams::v0).
// Round 0's verification cannot change an incoming state (one record per chunk: x_c is the
// predecessor's round-0 end), so every chunk is checked as soon as its own and its
// predecessor's walks are done: inside a tile by shuffle, across tiles by whichever of the
// two warps finishes second (tile-boundary arrival counters, no spinning).  A mismatch is
// recovered at once from x_c (Alg. 3 L16-18) with path fusion, exactly as the verify
// kernel's round-0 pass does; the counters go to the same pass slot.
// Returns bit 0 = hit, bit 1 = recovered (a task ran), bit 2 = the task moved the end;
// *cnt = the chunk's accept count on the true path (round-0 count, or the task's).
template <int MODE>
__device__ __forceinline__ uint32_t v0_check(const DevImage& img, const uint8_t* table, const RunParams& rp,
                                          const RecStore& rs, uint64_t c, uint32_t xin, uint32_t s0, uint32_t xo,
                                          uint32_t c0, uint32_t* cnt_out) {
  const bool hit = xin == s0;
  rs.found[c] = hit;
  if (rp.v0_chunk_ends) rp.v0_chunk_ends[c] = __ldg(img.inv + xo);  // speculative: exact unless a task moves an end
  if (hit) {
    *cnt_out = c0;
    return 1u;
  }
  uint32_t e, cnt;
  task_walk<MODE>(img, table, rp, rs, c, xin, &e, &cnt);
  const uint32_t ne = __ldcg(rs.n_end + c);
  const uint64_t o = (uint64_t)(ne % rp.vr_end) * rs.cap + c;
  __stcg(rs.start + o, xin);
  __stcg(rs.end + o, e);
  __stcg(rs.cnt + o, cnt);
  __stcg(rs.n_end + c, ne + 1);
  __stcg(rs.cur_end + c, e);
  *cnt_out = cnt;
  return 2u | (e != xo ? 4u : 0u);
}

// chunk c checked from the global record store (the other warp of its tile boundary)
template <int MODE>
__device__ __forceinline__ uint32_t v0_check_global(const DevImage& img, const uint8_t* table, const RunParams& rp,
                                                    const RecStore& rs, uint64_t c, uint32_t* cnt) {
  return v0_check<MODE>(img, table, rp, rs, c, __ldcg(rs.x + c), __ldcg(rs.start + c), __ldcg(rs.x + c + 1),
                        __ldcg(rs.cnt + c), cnt);
}

// atomicAdd with acquire-release semantics at GPU scope (PTX memory model): the release
// half publishes every write that happens-before it — the warp's lanes' record stores,
// ordered before lane 0 by __syncwarp — and the acquire half lets the second arrival read
// the first one's records; no full fence per tile.
__device__ __forceinline__ uint32_t atom_add_acq_rel(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}

__device__ __forceinline__ unsigned long long atom_add_acq_rel64(unsigned long long* p, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.add.acq_rel.gpu.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
  return old;
}

// per-warp fused-round-0 counters in shared memory (no registers held across the walk)
struct V0Sh {
  unsigned long long checks, matches, ntask, reread, ztot, fm;
  uint32_t tch, pad;
};

// The last warp of the spec kernel (all 32 lanes): commit round 0 as the verify kernel's
// round-0 pass would, and complete the run when no recovery changed an end (then the
// verify launch queued behind returns at once).  Lane 0 decides and clears the counters
// for the next run; the whole warp publishes the zero-copy result (one thread would
// serialise ~180 L2 reads).
__device__ __forceinline__ void v0_finalize(const RunParams& rp, const RecStore& rs, uint32_t lane) {
  Ctl* ctl = rp.v0_ctl;
  uint32_t finished = 0;
  if (lane == 0) {
    volatile Ctl* v = ctl;
    volatile unsigned long long* k = rs.v0c;
    const uint64_t N = rp.N;
    const uint64_t f2 = k[5] ? ~k[5] : N, nt = k[2];
    v->verify_checks = k[0];
    v->verify_matches = k[1];
    v->jacobi_iters = 1;
    v->fmin = f2;
    finished = f2 >= N;
    if (!finished) {  // commit round 1's tasks (the must-do is chunk f2)
      v->tasks_mustdo = 1;
      v->tasks_sre = nt - 1;
      v->reread_bytes = k[3];
      v->active_sum = nt;
      v->rounds = 1;
      v->f = f2;
      v->tf = __ldcg(rs.x + f2);
      if (k[6] == 0) {  // no task moved an end: round 1 verifies every chunk from f2
        v->verify_checks = v->verify_checks + (N - f2);
        v->verify_matches = v->verify_matches + (N - f2);
        v->fmin = N;
        finished = 1;
      }
    }
    if (finished) {
      v->accept_count = k[4];
      v->xfin = __ldcg(rs.x + N);
    }
    for (int i = 0; i < 8; i++) k[i] = 0;
    if (finished) v->finished = 1;
    __threadfence();
  }
  finished = __shfl_sync(0xffffffffu, finished, 0);
  if (finished && rp.h_out) {  // zero-copy result (as the verify kernel's finalize would publish it)
    const uint32_t* src = reinterpret_cast<const uint32_t*>(ctl);
    uint32_t* dst = reinterpret_cast<uint32_t*>(rp.h_out);
    for (uint32_t i = lane; i < sizeof(Ctl) / 4; i += 32) dst[i] = __ldcg(src + i);
  }
}

// TASKS = false: round 0 (starts from the lookback pair table).  TASKS = true: a dense
// recovery round (Alg. 3 L16-18 for many chunks at once): the round's task list
// (rs.task_chunk / rs.task_start, ntask entries, listed by the verification pass) is
// cut into groups of 32 tasks, one per lane; each stage gathers the 32 chunks' next
// 64 B with 8 TMA gather4 loads (tmap is then the {64 B x 1 row} gather map), so a
// round walks only the chunks that have a task.  Entries [0, nA) are A-tasks (must-do
// + SRE rear tasks: record to VR^end, the chunk's end moves); entries from nA on are
// RR / NF helper tasks (Alg. 4 L23-27, Alg. 5 L19-21): record to VR^others at the
// helper's precomputed ring position (oth_base[c] + task_j), nothing else changes.
// up to 28 warps (896 threads, 72 registers) for <= 8 paths per lane; 16 paths (CSE with
// spec_k 16: the whole lookback image of a 16-state convergence set) need 128 registers
template <int MODE, int KP, int S, bool TASKS, bool V0 = false>
__global__ void __launch_bounds__(KP > 8 ? 512 : 896, 1) k_spec_tma(const __grid_constant__ CUtensorMap tmap, DevImage img,
                                                    RunParams rp, RecStore rs, uint64_t n_full, uint32_t table_off,
                                                    uint64_t tile0, uint64_t f2, Ctl* ctl, uint64_t ntask) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // layout: [table (at offset 0: the lookup address is one IMAD)][stages: nwarps * S * 2 KiB][mbarriers]
  const uint32_t nwarps = blockDim.x / 32;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint8_t* table = smem_raw;
  uint8_t* stages = smem_raw + table_off;
  uint64_t* bars = reinterpret_cast<uint64_t*>(stages + (size_t)nwarps * S * kStageBytes);
  uint32_t* prow = reinterpret_cast<uint32_t*>(bars + ((nwarps * S + 1) & ~1u)) + warp * 32;  // TASKS: producer group's chunks
  stage_table(img, table);  // load-time data: staged before the dependency wait
  pdl_wait();                // the previous kernel in the stream (e.g. the last run's verify) is done
  uint64_t nA = 0;  // TASKS: entries [0, nA) of the list are A-tasks, the rest helpers
  if (TASKS) {  // device-driven dense round: the task list and frontier come from the control block
    if (!__ldcg(&ctl->dense_pending)) return;  // the verify launch before us handed no round over
    ntask = __ldcg(reinterpret_cast<const unsigned long long*>(&ctl->ntask[0]));
    f2 = __ldcg(reinterpret_cast<const unsigned long long*>(&ctl->fmin));
    nA = __ldcg(reinterpret_cast<const unsigned long long*>(&ctl->nA));
  }
  if (rp.ctl_init && blockIdx.x == 0) {
    init_ctl(rp.ctl_init, q0_of(rp), rp.N);
    if (rp.stamps && threadIdx.x == 0) rp.ctl_init->tl[0] = gtimer();
  }
  pdl_launch_dependents();   // the verify kernel may launch now; it waits for our completion
  if (lane == 0)
    for (int s = 0; s < S; s++) mbar_init(bars + warp * S + s, 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  using Sx = Step<MODE>;

  const uint32_t segs = rp.B / kRowBytes;
  const uint64_t ntiles = TASKS ? (ntask + 31) / 32 : (n_full + 31) / 32 - tile0;
  // TASKS: the task list may cover only part of the grid; warp-major numbering spreads
  // its groups over every SM (CTA-major would pack them into the first CTAs)
  const uint64_t gw = TASKS ? (uint64_t)warp * gridDim.x + blockIdx.x : (uint64_t)blockIdx.x * nwarps + warp;
  const uint64_t tw = (uint64_t)gridDim.x * nwarps;
  if (gw >= ntiles) return;
  struct StampEnd {  // timeline: the last warp to finish (profiling only)
    bool on; Ctl* c; uint32_t lane;
    __device__ ~StampEnd() {
      if (on && lane == 0) atomicMax(reinterpret_cast<unsigned long long*>(&c->tl[1]), (unsigned long long)gtimer());
    }
  } stamp_end{rp.stamps != 0 && rp.ctl_init != nullptr && !TASKS, rp.ctl_init, lane};
  const uint64_t my_tiles = (ntiles - gw + tw - 1) / tw;
  uint64_t n_mustdo = 0, n_sre = 0, n_hel = 0;
  bool helper = false;  // TASKS: this lane's task is a helper (VR^others)
  uint32_t hslot = 0;   // ... and its ring position in VR^others
  const uint64_t items = my_tiles * segs;  // (tile, segment) pairs streamed by this warp
  uint8_t* wst = stages + (size_t)warp * S * kStageBytes;
  uint64_t* wbar = bars + warp * S;

  // evict-first keeps a large table's cold rows in L2; a table that lives wholly in shared
  // memory (rp.tma_evict_normal) lets the input's 256 B lines stay until the warp's next
  // stages consume them (GSPEC_TMA_EVICT, A/B)
  const uint64_t pol = rp.tma_evict_normal ? evict_normal_policy() : evict_first_policy();
  // producer cursor (lane 0): the item S ahead of the consumer, tracked without divisions
  uint64_t p_tile = 0;
  uint32_t p_sg = 0, p_s = 0;
  auto issue_next = [&]() {  // called by every lane of the warp (lane 0 issues)
    const uint64_t t = tile0 + gw + p_tile * tw;
    if (TASKS && p_sg == 0) {  // new task group: its 32 chunks (the tail chunk / no task -> any full row)
      const uint64_t idx = t * 32 + lane;
      const uint32_t pc = idx < ntask ? __ldcg(rs.task_chunk + idx) : 0u;
      __syncwarp();
      prow[lane] = (uint32_t)min((uint64_t)pc, n_full - 1);
      __syncwarp();
    }
    if (lane == 0) {
      mbar_expect_tx(wbar + p_s, kStageBytes);
      if (TASKS) {
#pragma unroll
        for (int g = 0; g < 8; g++)
          tma_gather4(wst + (size_t)p_s * kStageBytes + g * 4 * kRowBytes, &tmap, wbar + p_s,
                      (int32_t)(p_sg * kRowBytes), reinterpret_cast<const uint4*>(prow)[g], pol);
      } else {
        tma_load_2d(wst + (size_t)p_s * kStageBytes, &tmap, wbar + p_s, (int32_t)(p_sg * kRowBytes),
                    (int32_t)(t * 32), pol);
      }
    }
    if (++p_sg == segs) { p_sg = 0; p_tile++; }
    if (++p_s == (uint32_t)S) p_s = 0;
  };
  for (uint64_t it = 0; it < items && it < (uint64_t)S; it++) issue_next();

  constexpr bool v0 = V0 && !TASKS && KP == 1;  // fused round-0 verification compiled in
  V0Sh* vsh = reinterpret_cast<V0Sh*>(prow + (blockDim.x / 32 - warp) * 32) + warp;  // after the prow block
  if (v0 && lane == 0) *vsh = V0Sh{0ull, 0ull, 0ull, 0ull, 0ull, ~0ull, 0u, 0u};
  uint32_t st[KP], code[KP], acc[KP], dacc[KP], kc = 1;
  bool single = false;  // spec-k: all paths of the warp's lanes merged (path fusion, P:427 [21])
  uint64_t c = 0, tile_i = 0;
  uint32_t sg = 0, s = 0, phase = 0;
  for (uint64_t it = 0; it < items; it++) {
    if (sg == 0) {  // new tile: predict this lane's chunk start (lookback-2 pair table)
      c = (tile0 + gw + tile_i * tw) * 32 + lane;
      if (TASKS) {  // c = this lane's task index until the chunk is known
        const uint64_t tix = c;
        const uint32_t tc = c < ntask ? __ldcg(rs.task_chunk + c) : 0xFFFFFFFFu;
        const uint32_t ts = (tc < n_full && tc >= f2) ? __ldcg(rs.task_start + c) : 0xFFFFFFFFu;
        c = tc;
        kc = ts != 0xFFFFFFFFu;  // 0: no task for this lane (walks a row's bytes, writes nothing)
        helper = tix >= nA;
        if (helper && kc) {
          const uint32_t j = __ldcg(rs.task_j + tix);
          // FIFO in task order (R16): a later helper of this round on the same chunk that
          // lands in the same ring slot evicts this record -> it is not stored (kNone)
          hslot = j + rp.vr_oth >= __ldcg(rs.hcnt + tc) ? (__ldcg(rs.oth_base + tc) + j) % rp.vr_oth : 0xFFFFFFFFu;
        }
#pragma unroll
        for (int p = 0; p < KP; p++) st[p] = kc ? ts : q0_of(rp);
      } else if (c == 0 || c >= n_full) {
        kc = 1;
#pragma unroll
        for (int p = 0; p < KP; p++) st[p] = q0_of(rp);
      } else {
        uint32_t ql;
        const uint32_t* qs = qs_chunk(img, rp, c, &ql);
        kc = min(rp.k, min(ql, rp.qs_cap));
#pragma unroll
        for (int p = 0; p < KP; p++) st[p] = __ldg(qs + min((uint32_t)p, kc - 1));
      }
#pragma unroll
      for (int p = 0; p < KP; p++) {
        code[p] = __ldg(img.tid2code + st[p]);
        acc[p] = 0;
        dacc[p] = 0;
      }
      single = false;
    }
    mbar_wait(wbar + s, phase);
    const uint8_t* row = wst + (size_t)s * kStageBytes + lane * kRowBytes;
    if (KP > 1 && single) {  // path fusion: every path of every lane has merged into path 0
#pragma unroll
      for (int u = 0; u < (int)(kRowBytes / 16); u++) {
        const uint4 q = *reinterpret_cast<const uint4*>(row + ((u ^ ((lane >> 1) & 3)) << 4));  // SWIZZLE_64B
        walk16<MODE>(img, table, q, code[0], acc[0]);
      }
    } else {
#pragma unroll
      for (int u = 0; u < (int)(kRowBytes / 16); u++) {
        const uint4 q = *reinterpret_cast<const uint4*>(row + ((u ^ ((lane >> 1) & 3)) << 4));  // SWIZZLE_64B
        if (KP == 1) {
          walk16<MODE>(img, table, q, code[0], acc[0]);
        } else {  // the paths share each symbol's class lookup
          const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
          for (int t = 0; t < 4; t++) {
            const uint32_t u1[1] = {w[t]};
            uint32_t k4[4];
            cls_words<MODE, 1>(img, table, u1, k4);
#pragma unroll
            for (int i = 0; i < 4; i++) {
#pragma unroll
              for (int p = 0; p < KP; p++) { code[p] = Sx::next(img, table, code[p], k4[i]); acc[p] += Sx::acc(code[p]); }
            }
          }
        }
      }
      if (KP > 1) {  // DFA determinism: paths that meet stay together; once all have met, walk one
        bool merged = true;
#pragma unroll
        for (int p = 1; p < KP; p++) merged = merged && code[p] == code[0];
        if (__all_sync(0xffffffffu, merged)) {
          single = true;
#pragma unroll
          for (int p = 0; p < KP; p++) dacc[p] = acc[p] - acc[0];
        }
      }
    }
    if (!TASKS && KP == 1 && rp.ck_shift && c < n_full) {  // R30: checkpoint of the round-0 path
      const uint32_t pe = (sg + 1) * kRowBytes;
      if ((pe & ((1u << rp.ck_shift) - 1u)) == 0 && pe < rp.B)
        rp.ck[(uint64_t)((pe >> rp.ck_shift) - 1) * rp.N + c] = make_uint2(code[0], acc[0]);
    }
    __syncwarp();
    if (it + S < items) issue_next();  // refill this stage
    if (TASKS && sg == segs - 1 && c < n_full && kc && helper) {  // helper done: append to VR^others
      if (hslot != 0xFFFFFFFFu) {
        const uint64_t o = (uint64_t)(kVrMax + hslot) * rs.cap + c;
        __stcg(rs.start + o, st[0]);
        __stcg(rs.end + o, Sx::tid(img, code[0]));
        __stcg(rs.cnt + o, acc[0]);
      }
      n_hel++;
    }
    if (TASKS && sg == segs - 1 && c < n_full && kc && !helper) {  // dense task done: append to VR^end
      const uint32_t e = Sx::tid(img, code[0]);
      const uint32_t ne = __ldcg(rs.n_end + c);
      const uint64_t o = (uint64_t)(ne % rp.vr_end) * rs.cap + c;
      __stcg(rs.start + o, st[0]);
      __stcg(rs.end + o, e);
      __stcg(rs.cnt + o, acc[0]);
      __stcg(rs.n_end + c, ne + 1);
      __stcg(rs.x + c + 1, e);  // Alg. 3 L17: the recovering chunk's end_c
      __stcg(rs.cur_end + c, e);
      if (c == f2) n_mustdo++; else n_sre++;
    }
    if (!TASKS && sg == segs - 1 && c < n_full) {  // tile done: round-0 records (VR^end)
      uint32_t e0 = 0;
#pragma unroll
      for (int p = 0; p < KP; p++) {
        const uint32_t e = Sx::tid(img, code[(KP > 1 && single) ? 0 : p]);
        if (p == 0) e0 = e;
        if ((uint32_t)p < kc) {
          rs.start[p * rs.cap + c] = st[p];
          rs.end[p * rs.cap + c] = e;
          rs.cnt[p * rs.cap + c] = (KP > 1 && single) ? acc[0] + dacc[p] : acc[p];
        }
      }
      rs.n_end[c] = kc;
      rs.n_oth[c] = 0;
      rs.next_qs[c] = (uint8_t)kc;
      rs.ref_start[c] = st[0];
      rs.ref_end[c] = e0;
      rs.ref_cnt[c] = acc[0];
      rs.x[c + 1] = e0;
      rs.cur_end[c] = e0;
      if (c == 0) rs.x[0] = q0_of(rp);
    }
    if (v0 && sg == segs - 1) {  // fused round-0 verification of this tile
      const bool mine = c < n_full;
      const uint32_t e_me = mine ? Sx::tid(img, code[0]) : 0u;
      const uint32_t prev = __shfl_up_sync(0xffffffffu, e_me, 1);
      uint32_t fl = 0, ct = 0;
      uint64_t fmc = ~0ull;
      if (mine && (lane > 0 || c == 0)) {
        fl = v0_check<MODE>(img, table, rp, rs, c, lane > 0 ? prev : q0_of(rp), st[0], e_me, acc[0], &ct);
        if (fl & 2u) fmc = c;
      }
      __syncwarp();  // the lanes' record stores happen-before lane 0's release below
      uint32_t xc = 0, xh = 0, xt = 0, xm = 0, ct2 = 0;  // lane 0: the boundary checks it ran
      if (lane == 0) {
        const uint64_t t = c / 32;  // this tile
        for (int side = 0; side < 2; side++) {
          const uint64_t tb = t + side;  // boundary tb: between tiles tb - 1 and tb
          const bool exists = side == 0 ? t > 0 : (t + 1) * 32 < n_full;
          if (!exists || !(atom_add_acq_rel(rp.v0_bflag + tb, 1u) & 1u)) continue;  // first: the other checks
          uint32_t cb = 0;
          const uint32_t f = v0_check_global<MODE>(img, table, rp, rs, tb * 32, &cb);
          xc++;
          xh += f & 1u;
          if (f & 2u) {
            xt++;
            fmc = min(fmc, (uint64_t)(tb * 32));
          }
          xm |= (f >> 2) & 1u;
          ct2 += cb;
        }
      }
      // tile totals -> the warp's shared counters (lane 0)
      const uint32_t chk = __popc(__ballot_sync(0xffffffffu, fl != 0));
      const uint32_t hits = __popc(__ballot_sync(0xffffffffu, fl & 1u));
      const uint32_t tasks = __popc(__ballot_sync(0xffffffffu, (fl & 2u) != 0));
      const uint32_t moved = __ballot_sync(0xffffffffu, (fl & 4u) != 0);
      uint32_t zs = ct;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        zs += __shfl_down_sync(0xffffffffu, zs, o);
        fmc = min(fmc, (uint64_t)__shfl_down_sync(0xffffffffu, (unsigned long long)fmc, o));
      }
      if (lane == 0) {
        vsh->checks += chk + xc;
        vsh->matches += hits + xh;
        vsh->ntask += tasks + xt;
        vsh->reread += (unsigned long long)(tasks + xt) * rp.B;
        vsh->ztot += (unsigned long long)zs + ct2;
        vsh->fm = min(vsh->fm, (unsigned long long)fmc);
        vsh->tch |= (moved != 0) | xm;
      }
      __syncwarp();
    }
    if (++sg == segs) { sg = 0; tile_i++; }
    if (++s == (uint32_t)S) { s = 0; phase ^= 1u; }
  }
  if (v0) {  // fused round 0: the warp's counters; the last warp finalises
    uint32_t last = 0;
    if (lane == 0) {
      unsigned long long* k = rs.v0c;
      const unsigned long long w[5] = {vsh->checks, vsh->matches, vsh->ntask, vsh->reread, vsh->ztot};
      for (int i = 0; i < 5; i++)
        if (w[i]) atomicAdd(k + i, w[i]);
      if (vsh->fm != ~0ull) atomicMax(k + 5, ~vsh->fm);  // ~chunk: the largest is the first task chunk
      if (vsh->tch) atomicOr(k + 6, 1ull);
      const uint64_t warps = min(ntiles, tw);  // warps that walk tiles
      last = atom_add_acq_rel64(k + 7, 1ull) == warps - 1;
    }
    if (__shfl_sync(0xffffffffu, last, 0)) v0_finalize(rp, rs, lane);
  }
  if (TASKS) {  // warp-level stats (warps may have returned early: no block barrier here)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      n_mustdo += __shfl_down_sync(0xffffffffu, n_mustdo, o);
      n_sre += __shfl_down_sync(0xffffffffu, n_sre, o);
      n_hel += __shfl_down_sync(0xffffffffu, n_hel, o);
    }
    if (lane == 0 && n_mustdo + n_sre + n_hel) {
      atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->tasks_mustdo), (unsigned long long)n_mustdo);
      atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->tasks_sre), (unsigned long long)n_sre);
      if (n_hel) atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->tasks_helper), (unsigned long long)n_hel);
      atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->active_sum),
                (unsigned long long)(n_mustdo + n_sre + n_hel));
      atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->reread_bytes),
                (unsigned long long)((n_mustdo + n_sre + n_hel) * rp.B));
      atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->walked_bytes),
                (unsigned long long)((n_mustdo + n_sre + n_hel) * rp.B));
    }
  }
}

// Checkpointed dense recovery round (R30), one segment pass.  The same task list
// and records as k_spec_tma<TASKS>, but a task stops as soon as its path meets the chunk's
// round-0 path at a checkpoint (rp.ck, written by the round-0 walk every 2^ck_shift bytes):
// by determinism the rest of the path is the round-0 path, so end = ref_end and count =
// (the task's count so far) + (ref_cnt - the round-0 count at the checkpoint).  A warp's
// lanes step together, so a lane that stops early only idles; the round is therefore cut
// into passes over byte segments [pass * seg, (pass + 1) * seg) of the chunks: pass 0 walks
// every task of the list over the first segment, and the tasks still running at its end
// are appended (task, code, count) to a compact list that pass 1 walks over the next
// segment, and so on — every pass starts with full warps.  Every chain of a pass is at the
// same byte offset, so a stage is still 8 TMA gather4 loads of one 64 B column of 32 chunks.
// Counters: segn[p % 3] = entries appended by pass p (pass p clears segn[(p + 1) % 3], the
// finish kernel all three).
struct SegEntry {
  uint32_t t, code, acc, pad;
};

// RB: bytes of a chunk per stage (64: SWIZZLE_64B boxes; 128: SWIZZLE_128B, half the TMA
// issue work per byte — 8 gather4 loads per stage either way)
template <int MODE, int S, int RB>
__global__ void __launch_bounds__(896, 1) k_task_seg(const __grid_constant__ CUtensorMap tmap, DevImage img,
                                                     RunParams rp, RecStore rs, uint64_t n_full, uint32_t table_off,
                                                     Ctl* ctl, uint32_t pass, uint32_t seg, SegEntry* seg_list,
                                                     uint32_t commit) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  constexpr uint32_t kRowB = RB, kStB = 32 * RB;
  const uint32_t nwarps = blockDim.x / 32;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint8_t* table = smem_raw;
  uint8_t* stages = smem_raw + table_off;
  uint64_t* bars = reinterpret_cast<uint64_t*>(stages + (size_t)nwarps * S * kStB);
  uint32_t* prow = reinterpret_cast<uint32_t*>(bars + ((nwarps * S + 1) & ~1u)) + warp * 32;
  stage_table(img, table);
  pdl_wait();
  if (!__ldcg(&ctl->dense_pending)) return;  // spare slot: the run needs no dense round
  const uint32_t B = rp.B;
  const uint32_t x0 = pass * seg, x1 = min(B, x0 + seg);
  if (x0 >= B) return;
  const uint64_t ntask = __ldcg(reinterpret_cast<const unsigned long long*>(&ctl->ntask[0]));
  const uint64_t f2 = __ldcg(reinterpret_cast<const unsigned long long*>(&ctl->fmin));
  const uint64_t nA = __ldcg(reinterpret_cast<const unsigned long long*>(&ctl->nA));
  const uint64_t cap = rs.cap;
  const SegEntry* in_list = seg_list + (uint64_t)((pass + 1) & 1) * cap;  // written by pass - 1
  SegEntry* out_list = seg_list + (uint64_t)(pass & 1) * cap;
  const uint64_t n_in = pass == 0 ? ntask : (uint64_t)__ldcg(&ctl->segn[(pass + 2) % 3]);
  if (n_in > cap) __trap();
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->segn[(pass + 1) % 3] = 0;  // pass + 1's output
  pdl_launch_dependents();
  const uint64_t ngroups = (n_in + 31) / 32;
  const uint64_t gw = (uint64_t)warp * gridDim.x + blockIdx.x, tw = (uint64_t)gridDim.x * nwarps;
  // (no block barrier below: warps are independent; a warp without a group walks nothing but
  // still takes its commit ticket)
  if (lane == 0)
    for (int s = 0; s < S; s++) mbar_init(bars + warp * S + s, 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();
  using Sx = Step<MODE>;
  uint8_t* wst = stages + (size_t)warp * S * kStB;
  uint64_t* wbar = bars + warp * S;
  const uint64_t pol = evict_first_policy();
  const uint32_t ckm = (1u << rp.ck_shift) - 1u;
  const uint32_t segs = (x1 - x0) / kRowB;
  const uint64_t my_groups = gw < ngroups ? (ngroups - gw + tw - 1) / tw : 0;
  const uint64_t items = my_groups * segs;
  unsigned long long n_mustdo = 0, n_sre = 0, n_hel = 0, walked = 0;

  uint64_t p_group = 0;
  uint32_t p_sg = 0, p_s = 0;
  auto issue_next = [&]() {  // every lane of the warp (lane 0 issues)
    if (p_sg == 0) {  // new group: its 32 chunks
      const uint64_t idx = (gw + p_group * tw) * 32 + lane;
      uint32_t pc = 0;
      if (idx < n_in) {
        const uint32_t t = pass == 0 ? (uint32_t)idx : __ldcg(&in_list[idx].t);
        pc = __ldcg(rs.task_chunk + t);
      }
      __syncwarp();
      prow[lane] = (uint32_t)min((uint64_t)pc, n_full - 1);
      __syncwarp();
    }
    if (lane == 0) {
      mbar_expect_tx(wbar + p_s, kStB);
#pragma unroll
      for (int g = 0; g < 8; g++)
        tma_gather4(wst + (size_t)p_s * kStB + g * 4 * kRowB, &tmap, wbar + p_s, (int32_t)(x0 + p_sg * kRowB),
                    reinterpret_cast<const uint4*>(prow)[g], pol);
    }
    if (++p_sg == segs) { p_sg = 0; p_group++; }
    if (++p_s == (uint32_t)S) p_s = 0;
  };
  for (uint64_t it = 0; it < items && it < (uint64_t)S; it++) issue_next();

  uint32_t t = 0, c = 0, st0 = 0, code = 0, acc = 0;
  bool live = false;  // this lane's chain still walks
  uint64_t group_i = 0;
  uint32_t sg = 0, s = 0, phase = 0;
  for (uint64_t it = 0; it < items; it++) {
    if (sg == 0) {  // new group: this lane's chain
      const uint64_t idx = (gw + group_i * tw) * 32 + lane;
      live = false;
      code = __ldg(img.tid2code + q0_of(rp));  // any valid code for an idle lane
      acc = 0;
      if (idx < n_in) {
        if (pass == 0) {
          t = (uint32_t)idx;
          c = __ldcg(rs.task_chunk + t);
          st0 = (c < n_full && c >= f2) ? __ldcg(rs.task_start + t) : kNoTask;
          if (st0 != kNoTask) {
            live = true;
            code = __ldg(img.tid2code + st0);
          }
        } else {
          const SegEntry e = in_list[idx];
          t = e.t;
          c = __ldcg(rs.task_chunk + t);
          st0 = __ldcg(rs.task_start + t);
          // guards (compute-sanitizer is unavailable on the GPU pool; a violated bound traps)
          if (idx >= cap || t >= ntask || c < f2 || c >= n_full) __trap();
          code = e.code;
          acc = e.acc;
          live = true;
        }
      }
    }
    mbar_wait(wbar + s, phase);
    uint32_t k = code, a = acc;
    const uint8_t* row = wst + (size_t)s * kStB + lane * kRowB;
#pragma unroll
    for (int u = 0; u < (int)(kRowB / 16); u++) {  // SWIZZLE_64B / SWIZZLE_128B: chunk u ^ (row bits)
      const uint32_t sw = RB == 64 ? ((lane >> 1) & 3) : (lane & 7);
      const uint4 q = *reinterpret_cast<const uint4*>(row + ((u ^ sw) << 4));
      walk16<MODE>(img, table, q, k, a);
    }
    __syncwarp();
    if (it + S < items) issue_next();  // refill this stage
    if (live) {
      code = k;
      acc = a;
      walked += kRowB;
      const uint32_t pe = x0 + (sg + 1) * kRowB;
      bool fin = false;
      uint32_t e = 0, cnt = 0;
      if (pe >= B) {
        fin = true;
        e = Sx::tid(img, code);
        cnt = acc;
      } else if ((pe & ckm) == 0) {
        const uint2 ck = __ldcg(rp.ck + (uint64_t)((pe >> rp.ck_shift) - 1) * rp.N + c);
        if (ck.x == code) {  // met the round-0 path: the rest of the chunk is its path
          fin = true;
          e = __ldcg(rs.ref_end + c);
          cnt = acc + (__ldcg(rs.ref_cnt + c) - ck.y);
        }
      }
      if (fin) {
        live = false;
        if (t >= nA) {  // RR / NF helper: VR^others at its precomputed ring slot
          const uint32_t j = __ldcg(rs.task_j + t);
          if (j + rp.vr_oth >= __ldcg(rs.hcnt + c)) {  // not evicted within its own round (R16)
            const uint64_t o = (uint64_t)(kVrMax + (__ldcg(rs.oth_base + c) + j) % rp.vr_oth) * rs.cap + c;
            __stcg(rs.start + o, st0);
            __stcg(rs.end + o, e);
            __stcg(rs.cnt + o, cnt);
          }
          n_hel++;
        } else {  // A-task: VR^end, the chunk's end moves (Alg. 3 L17)
          const uint32_t ne = __ldcg(rs.n_end + c);
          const uint64_t o = (uint64_t)(ne % rp.vr_end) * rs.cap + c;
          __stcg(rs.start + o, st0);
          __stcg(rs.end + o, e);
          __stcg(rs.cnt + o, cnt);
          __stcg(rs.n_end + c, ne + 1);
          __stcg(rs.x + c + 1, e);
          __stcg(rs.cur_end + c, e);
          if (c == f2) n_mustdo++; else n_sre++;
        }
      }
    }
    if (sg == segs - 1) {  // segment done: the chains still walking go to the next pass's list
      const uint32_t m = __ballot_sync(0xffffffffu, live);
      if (m) {
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(&ctl->segn[pass % 3], (uint32_t)__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (live) {
          const uint32_t o = base + __popc(m & ((1u << lane) - 1u));
          if (o >= n_in || o >= cap) __trap();  // a pass never appends more chains than it read
          out_list[o] = SegEntry{t, code, acc, 0u};
        }
      }
    }
    if (++sg == segs) { sg = 0; group_i++; }
    if (++s == (uint32_t)S) { s = 0; phase ^= 1u; }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    n_mustdo += __shfl_down_sync(0xffffffffu, n_mustdo, o);
    n_sre += __shfl_down_sync(0xffffffffu, n_sre, o);
    n_hel += __shfl_down_sync(0xffffffffu, n_hel, o);
    walked += __shfl_down_sync(0xffffffffu, walked, o);
  }
  if (lane == 0 && n_mustdo + n_sre + n_hel + walked) {
    atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->tasks_mustdo), n_mustdo);
    atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->tasks_sre), n_sre);
    if (n_hel) atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->tasks_helper), n_hel);
    atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->active_sum), n_mustdo + n_sre + n_hel);
    atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->reread_bytes), (n_mustdo + n_sre + n_hel) * B);
    atomicAdd(reinterpret_cast<unsigned long long*>(&ctl->walked_bytes), walked);
  }
  if (commit) {  // last pass, no tail chunk: the last warp commits the round (the finish kernel's job)
    uint32_t last = 0;
    if (lane == 0) {
      __threadfence();
      last = atomicAdd(&ctl->seg_done, 1u) == gridDim.x * nwarps - 1;
    }
    if (__shfl_sync(0xffffffffu, last, 0) && lane == 0) {
      __threadfence();
      ctl->segn[0] = ctl->segn[1] = ctl->segn[2] = 0;
      ctl->rounds++;
      ctl->dense_rounds++;
      ctl->f = f2;
      ctl->tf = __ldcg(rs.x + f2);
      ctl->changed[0] = 0;  // the verify launch behind us starts its passes at slot 0
      ctl->it_fm[0] = rp.N;
      ctl->it_checks[0] = ctl->it_matches[0] = ctl->it_ntask[0] = ctl->it_reread[0] = 0;
      ctl->seg_done = 0;
      __threadfence();
      ctl->dense_pending = 0;
    }
  }
}

using EncodeFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                              const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                              CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeFn get_encode() {
  static EncodeFn fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeFn>(p);
  }
  return fn;
}

// Pick warps per CTA (one CTA per SM) so the tile count divides evenly over
// the resident warps (wave quantization), within the smem budget.
uint32_t pick_warps(uint64_t ntiles, int sms, uint32_t wmax) {
  uint32_t best = wmax;
  double best_score = -1;
  for (uint32_t w = 8; w <= wmax; w++) {
    const double slots = (double)sms * w;
    const double rounds = std::ceil((double)ntiles / slots);
    const double eff = (double)ntiles / (rounds * slots);
    const double score = eff * std::min(1.0, w / 24.0);  // ~24 one-chain warps hide the lookup latency
    if (score > best_score + 1e-9) { best_score = score; best = w; }
  }
  return best;
}

template <int MODE, int KP, int S, bool TASKS, bool V0 = false>
cudaError_t launch_tma_t(const CUtensorMap& tm, const DevImage& img, const RunParams& rp, const RecStore& rs,
                         uint64_t n_full, int sms, cudaStream_t st, uint64_t tile0, uint64_t f2, Ctl* ctl,
                         uint64_t ntask) {
  auto kern = k_spec_tma<MODE, KP, S, TASKS, V0>;
  const uint64_t ntiles = TASKS ? (ntask + 31) / 32 : (n_full + 31) / 32 - tile0;
  if (ntiles == 0) return cudaSuccess;
  const uint32_t tbytes = smem_bytes_for(img);
  const uint32_t per_warp = S * kStageBytes + S * 8 + 128 + 64;
  const uint32_t avail = 227 * 1024 - ((tbytes + 1023) & ~1023u) - 64;
  uint32_t wmax = std::min<uint32_t>(KP > 8 ? 16 : 28, avail / per_warp);  // launch bounds 896 / 512
  if (wmax < 4) return cudaErrorInvalidConfiguration;
  uint32_t w = pick_warps(ntiles, sms, wmax);
  if (wmax < 8) w = wmax;
  const uint32_t table_off = (tbytes + 1023) & ~1023u;  // stages start 1 KiB-aligned (swizzle span)
  const uint32_t smem = table_off + w * S * kStageBytes + ((w * S + 1) & ~1u) * 8 + w * 128 + w * 64;
  cudaError_t e = kernel_setup((const void*)kern, smem, (int)(w * 32), nullptr);
  if (e != cudaSuccess) return e;
  uint64_t grid = std::min<uint64_t>((uint64_t)sms, (ntiles + w - 1) / w);
  if (grid < 1) grid = 1;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(w * 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, tm, img, rp, rs, n_full, table_off, tile0, f2, ctl, ntask);
}

template <int MODE, int KP, bool TASKS, bool V0 = false>
cudaError_t launch_tma_s(const CUtensorMap& tm, const DevImage& img, const RunParams& rp, const RecStore& rs,
                         uint64_t n_full, int sms, cudaStream_t st, uint64_t tile0, uint64_t f2, Ctl* ctl,
                         uint64_t ntask = 0) {
  const uint32_t tbytes = smem_bytes_for(img);
  if (tbytes + 24 * (3 * kStageBytes) + 2048 + 24 * 128 <= 227 * 1024)
    return launch_tma_t<MODE, KP, 3, TASKS, V0>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask);
  return launch_tma_t<MODE, KP, 2, TASKS, V0>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask);
}

template <int MODE>
cudaError_t launch_tma_m(const CUtensorMap& tm, const DevImage& img, const RunParams& rp, const RecStore& rs,
                         uint64_t n_full, int sms, cudaStream_t st) {
  if (rp.k <= 1 && rp.v0) return launch_tma_s<MODE, 1, false, true>(tm, img, rp, rs, n_full, sms, st, 0, 0, nullptr);
  if (rp.k <= 1) return launch_tma_s<MODE, 1, false>(tm, img, rp, rs, n_full, sms, st, 0, 0, nullptr);
  if (rp.k <= 2) return launch_tma_s<MODE, 2, false>(tm, img, rp, rs, n_full, sms, st, 0, 0, nullptr);
  if (rp.k <= 4) return launch_tma_s<MODE, 4, false>(tm, img, rp, rs, n_full, sms, st, 0, 0, nullptr);
  if (rp.k <= 8) return launch_tma_s<MODE, 8, false>(tm, img, rp, rs, n_full, sms, st, 0, 0, nullptr);
  return launch_tma_s<MODE, 16, false>(tm, img, rp, rs, n_full, sms, st, 0, 0, nullptr);
}

// R30: the segment passes of a checkpointed dense round (one CTA per SM, warps chosen as
// for the task kernel; each pass reads its list length on the device)
template <int MODE, int S, int RB>
cudaError_t launch_seg_t(const CUtensorMap& tm, const DevImage& img, const RunParams& rp, const RecStore& rs,
                         uint64_t n_full, int sms, cudaStream_t st, Ctl* ctl, uint32_t seg, void* seg_list,
                         bool commit_last, uint32_t pass) {
  auto kern = k_task_seg<MODE, S, RB>;
  constexpr uint32_t kStB = 32 * RB;
  const uint32_t tbytes = smem_bytes_for(img);
  const uint32_t per_warp = S * kStB + S * 8 + 128;
  const uint32_t avail = 227 * 1024 - ((tbytes + 1023) & ~1023u) - 64;
  uint32_t w = std::min<uint32_t>(28, avail / per_warp);
  if (const char* ev = getenv("GSPEC_CK_WARPS")) w = std::min<uint32_t>(w, (uint32_t)std::max(4, atoi(ev)));
  if (w < 4) return cudaErrorInvalidConfiguration;
  const uint32_t table_off = (tbytes + 1023) & ~1023u;
  const uint32_t smem = table_off + w * S * kStB + ((w * S + 1) & ~1u) * 8 + w * 128;
  cudaError_t e = kernel_setup((const void*)kern, smem, (int)(w * 32), nullptr);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)sms);
  cfg.blockDim = dim3(w * 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  const uint32_t passes = (rp.B + seg - 1) / seg;
  return cudaLaunchKernelEx(&cfg, kern, tm, img, rp, rs, n_full, table_off, ctl, pass, seg,
                            reinterpret_cast<SegEntry*>(seg_list), (uint32_t)(commit_last && pass + 1 == passes));
}

template <int MODE>
cudaError_t launch_seg_s(const CUtensorMap& tm, const CUtensorMap& tm128, bool r128, const DevImage& img,
                         const RunParams& rp, const RecStore& rs, uint64_t n_full, int sms, cudaStream_t st, Ctl* ctl,
                         uint32_t seg, void* seg_list, bool commit_last) {
  const uint32_t tbytes = smem_bytes_for(img);
  const bool s3 = tbytes + 24 * (3 * kStageBytes) + 2048 + 24 * 128 <= 227 * 1024;
  const uint32_t passes = (rp.B + seg - 1) / seg;
  for (uint32_t p = 0; p < passes; p++) {
    cudaError_t e;
    // pass 0 (every task: bound by the shared pipe) keeps 64 B rows and the most warps; the later
    // passes (fewer chains: bound by a warp's issue latency) take 128 B rows, half the TMA issue
    // work per byte (R30)
    if (p > 0 && r128)
      e = launch_seg_t<MODE, 2, 128>(tm128, img, rp, rs, n_full, sms, st, ctl, seg, seg_list, commit_last, p);
    else if (s3)
      e = launch_seg_t<MODE, 3, 64>(tm, img, rp, rs, n_full, sms, st, ctl, seg, seg_list, commit_last, p);
    else
      e = launch_seg_t<MODE, 2, 64>(tm, img, rp, rs, n_full, sms, st, ctl, seg, seg_list, commit_last, p);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// gather = false: box {64 B, 32 chunks} (tiles of consecutive chunks);
// gather = true: box {64 B, 1 chunk} for tile::gather4 (4 arbitrary chunks per load)
bool encode_map(const RunParams& rp, uint64_t n_full, CUtensorMap* tm, bool gather = false, uint32_t rowb = kRowBytes) {
  EncodeFn enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {rp.B, n_full};
  cuuint64_t strides[1] = {rp.B};
  cuuint32_t box[2] = {rowb, gather ? 1u : 32u};
  cuuint32_t es[2] = {1, 1};
  return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<uint8_t*>(rp.in), dims, strides, box, es,
             CU_TENSOR_MAP_INTERLEAVE_NONE, rowb == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B,
             tma_promotion() == 1 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
             : tma_promotion() == 2 ? CU_TENSOR_MAP_L2_PROMOTION_NONE : CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool tma_applies(const RunParams& rp, uint64_t n_full) {
  return n_full > 0 && rp.B % kRowBytes == 0 && (reinterpret_cast<uintptr_t>(rp.in) & 15u) == 0 &&
         n_full < (1ull << 31);
}

}  // namespace

// Returns cudaErrorNotSupported when the TMA path does not apply (caller falls
// back to the generic kernel): unaligned input, B % 64 != 0, no full chunks.
cudaError_t launch_spec_tma(const DevImage& img, const RunParams& rp, const RecStore& rs, int sms, cudaStream_t st,
                            uint64_t* n_done) {
  *n_done = 0;
  const uint64_t n_full = rp.len / rp.B;
  CUtensorMap tm;
  if (!tma_applies(rp, n_full) || !encode_map(rp, n_full, &tm)) return cudaErrorNotSupported;
  cudaError_t e;
  switch (img.mode) {
    case MODE_U8: e = launch_tma_m<MODE_U8>(tm, img, rp, rs, n_full, sms, st); break;
    case MODE_U16: e = launch_tma_m<MODE_U16>(tm, img, rp, rs, n_full, sms, st); break;
    case MODE_U16H: e = launch_tma_m<MODE_U16H>(tm, img, rp, rs, n_full, sms, st); break;
    case MODE_U16D:
      e = img.delta_exc == 1 ? launch_tma_m<MODE_U16D1>(tm, img, rp, rs, n_full, sms, st)
                             : launch_tma_m<MODE_U16D>(tm, img, rp, rs, n_full, sms, st);
      break;
    default: e = launch_tma_m<MODE_U32>(tm, img, rp, rs, n_full, sms, st); break;
  }
  if (e == cudaSuccess) *n_done = n_full;
  return e;
}

// Dense recovery round over the task list (ctl->ntask[0] entries, read on the device):
// chunks < n_full are walked here; the tail chunk (if its task is listed) is left to the
// finish kernel.  Launched with the grid of a full list (one CTA per SM, persistent).
cudaError_t launch_task_tma(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* ctl, int sms,
                            cudaStream_t st, uint64_t* n_done, bool* committed) {
  *n_done = 0;
  if (committed) *committed = false;
  const uint64_t n_full = rp.len / rp.B;
  CUtensorMap tm;
  if (rp.ck_shift && rp.ck_seg && tma_applies(rp, n_full) && encode_map(rp, n_full, &tm, true)) {  // R30
    cudaError_t e;
    const uint32_t sg = rp.ck_seg;
    const bool cm = n_full == rp.N;  // no tail chunk: the last pass commits, no finish kernel
    // 128 B rows when the chunk, the segment and the checkpoint interval are multiples of 128 and
    // two 4 KiB stages per warp leave room for >= 16 warps beside the table (GSPEC_CK_ROW=64: off)
    CUtensorMap tm128;
    static int row_env = -1;
    if (row_env < 0) {
      const char* e = getenv("GSPEC_CK_ROW");
      row_env = e ? atoi(e) : 128;
    }
    const bool r128 = row_env == 128 && rp.B % 128 == 0 && sg % 128 == 0 && (1u << rp.ck_shift) % 128 == 0 &&
                      smem_bytes_for(img) + 16 * (2 * 4096 + 16 + 128) + 2048 <= 227 * 1024 &&
                      encode_map(rp, n_full, &tm128, true, 128);
    if (committed) *committed = cm;
    switch (img.mode) {
      case MODE_U8: e = launch_seg_s<MODE_U8>(tm, tm128, r128, img, rp, rs, n_full, sms, st, ctl, sg, rp.ck_list, cm); break;
      case MODE_U16: e = launch_seg_s<MODE_U16>(tm, tm128, r128, img, rp, rs, n_full, sms, st, ctl, sg, rp.ck_list, cm); break;
      case MODE_U16H: e = launch_seg_s<MODE_U16H>(tm, tm128, r128, img, rp, rs, n_full, sms, st, ctl, sg, rp.ck_list, cm); break;
      case MODE_U16D:
        e = img.delta_exc == 1 ? launch_seg_s<MODE_U16D1>(tm, tm128, r128, img, rp, rs, n_full, sms, st, ctl, sg, rp.ck_list, cm)
                               : launch_seg_s<MODE_U16D>(tm, tm128, r128, img, rp, rs, n_full, sms, st, ctl, sg, rp.ck_list, cm);
        break;
      default: e = launch_seg_s<MODE_U32>(tm, tm128, r128, img, rp, rs, n_full, sms, st, ctl, sg, rp.ck_list, cm); break;
    }
    if (e == cudaSuccess) *n_done = n_full;
    return e;
  }
  if (!tma_applies(rp, n_full) || !encode_map(rp, n_full, &tm, true)) return cudaErrorNotSupported;
  const uint64_t tile0 = 0, f2 = 0, ntask = n_full;  // launch-shape hints; the kernel reads the real values
  cudaError_t e;
  switch (img.mode) {
    case MODE_U8: e = launch_tma_s<MODE_U8, 1, true>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask); break;
    case MODE_U16: e = launch_tma_s<MODE_U16, 1, true>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask); break;
    case MODE_U16H: e = launch_tma_s<MODE_U16H, 1, true>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask); break;
    case MODE_U16D:
      e = img.delta_exc == 1 ? launch_tma_s<MODE_U16D1, 1, true>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask)
                             : launch_tma_s<MODE_U16D, 1, true>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask);
      break;
    default: e = launch_tma_s<MODE_U32, 1, true>(tm, img, rp, rs, n_full, sms, st, tile0, f2, ctl, ntask); break;
  }
  if (e == cudaSuccess) *n_done = n_full;
  return e;
}

}  // namespace gspec
