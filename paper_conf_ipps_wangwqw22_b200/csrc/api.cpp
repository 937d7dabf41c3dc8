// api.cpp — the C ABI of include/gspec.h: DFA preparation (frequency-based
// transformation, byte classes, packing), the run driver (spec exec
// -> verify/recover rounds -> finalize), ENUM, the scheme selector.
// Host code only; every step of the hot path runs in the sm_100a kernels.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <map>
#include <numeric>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "gspec.h"
#include "internal.h"

using namespace gspec;

namespace {

thread_local std::string g_err;

int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

#define CUDA_TRY(expr)                                                                         \
  do {                                                                                         \
    cudaError_t _e = (expr);                                                                   \
    if (_e != cudaSuccess)                                                                     \
      return fail(_e == cudaErrorMemoryAllocation ? FSM_ENOMEM : FSM_ECUDA,                    \
                  std::string(#expr) + ": " + cudaGetErrorString(_e));                         \
  } while (0)

int dev_alloc(fsm_t f, void** p, size_t bytes) {
  cudaError_t e = cudaMalloc(p, bytes ? bytes : 16);
  if (e != cudaSuccess) return fail(FSM_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
  f->owned.push_back(*p);
  return FSM_OK;
}

template <typename T>
int upload(fsm_t f, const T** dst, const std::vector<T>& v, size_t pad_bytes = 0) {
  void* p = nullptr;
  const size_t bytes = v.size() * sizeof(T);
  int rc = dev_alloc(f, &p, bytes + pad_bytes + 16);
  if (rc) return rc;
  CUDA_TRY(cudaMemset(p, 0, bytes + pad_bytes + 16));
  if (bytes) CUDA_TRY(cudaMemcpy(p, v.data(), bytes, cudaMemcpyHostToDevice));
  *dst = reinterpret_cast<const T*>(p);
  return FSM_OK;
}

// Every entry point starts by clearing a stale (non-sticky) CUDA error left by a
// failed runtime call elsewhere in this thread, so it is not reported by our own
// launch checks; GSPEC_DEBUG_ERR=1 prints it.
void entry_clear(const char* name) {
  const cudaError_t e = cudaGetLastError();
  static const bool dbg = getenv("GSPEC_DEBUG_ERR") != nullptr;
  if (e != cudaSuccess && dbg) fprintf(stderr, "gspec: stale CUDA error at %s entry: %s\n", name, cudaGetErrorString(e));
}

// One NVTX range per C-ABI call (tracing: nsys / ncu --nvtx show which entry point and
// phase enqueued each kernel); NVTX v3 is header-only and a no-op without a tool attached.
struct ApiScope {
  explicit ApiScope(const char* name) {
    entry_clear(name);
    nvtxRangePushA(name);
  }
  ~ApiScope() { nvtxRangePop(); }
};

struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

constexpr uint32_t kRow8Bytes = 260;  // walk.cuh kRow8: row r starts at bank (r * 65) % 32 = r % 32

// MODE_U8 row placement from a profile sample (an extension of the transformation,
// DESIGN.md §5.1): the lanes of a warp walk different chunks, so one warp-wide
// lookup reads up to 32 rows; two lanes conflict when their (row, byte) words
// fall in one bank.  Rows of frequently visited states are given codes (row
// numbers, accept flag in bit 7) whose bank rotation keeps their hot words off
// the banks already loaded by hotter rows: greedy over states by visits, cost =
// sum over the state's word histogram of the bank load so far.  Codes are
// drawn from [0, n_na + 32) and [128, 128 + n_acc + 32) so every rotation is
// available at a bounded table size.  Purely a layout choice: tids, the
// transformation and all results are unchanged.
void place_rows_bank_aware(fsm_t f, const std::vector<uint32_t>& ttc, uint32_t C, const std::vector<uint8_t>& acc_t,
                           uint32_t n_na, uint32_t n_acc, const uint8_t* sample, uint64_t len,
                           std::vector<uint32_t>& tid2code, std::vector<uint32_t>& code2tid) {
  const uint32_t nt = f->n + 1, P = f->n;
  std::vector<double> visits(nt, 0.0), hist((size_t)nt * 64, 0.0);
  uint32_t t = f->perm[f->q0];
  for (uint64_t i = 0; i < len; i++) {
    const uint8_t b = sample[i];
    visits[t] += 1;
    hist[(size_t)t * 64 + (b >> 2)] += 1;
    t = t == P ? P : ttc[(uint64_t)t * C + f->cls[b]];
  }
  std::vector<uint32_t> order(nt);
  std::iota(order.begin(), order.end(), 0u);
  std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return visits[a] > visits[b]; });
  std::vector<uint8_t> used(256, 0);
  const uint32_t lim_na = std::min(128u, n_na + 32), lim_acc = std::min(256u, 128 + n_acc + 32);
  double load[32] = {0};
  for (uint32_t q : order) {
    const uint32_t lo = acc_t[q] ? 128 : 0, hi = acc_t[q] ? lim_acc : lim_na;
    uint32_t best = 256;
    double best_cost = 0;
    for (uint32_t c = lo; c < hi; c++) {
      if (used[c]) continue;
      double cost = 0;
      if (visits[q] > 0)
        for (uint32_t w = 0; w < 64; w++) cost += hist[(size_t)q * 64 + w] * load[(w + c) % 32];
      if (best == 256 || cost < best_cost) { best = c; best_cost = cost; }
      if (visits[q] == 0) break;  // never visited: first free code
    }
    used[best] = 1;
    tid2code[q] = best;
    code2tid[best] = q;
    for (uint32_t w = 0; w < 64; w++) load[(w + best) % 32] += hist[(size_t)q * 64 + w];
  }
}

// ENUM sub-chunk size E | B: halve down to 256 B while the map count stays <= 4 M (measured
// on C1: going further, to 64 B, made the scan levels cost more than the walk saved).
uint32_t enum_sub_bytes(uint32_t B, uint64_t len) {
  uint32_t E = B;
  while (E % 32 == 0 && E > 256 && (len + E / 2 - 1) / (E / 2) <= (1ull << 22)) E /= 2;
  return E;
}

struct Opts {
  fsm_scheme scheme;
  uint32_t B, k, k_cse, L, qs_cap, vr_end, vr_oth;
  cudaStream_t st;
};

int resolve_opts(const fsm_run_opts* o, Opts* r) {
  r->scheme = o ? o->scheme : FSM_SCHEME_AUTO;
  r->B = (o && o->chunk_bytes) ? o->chunk_bytes : 4096;
  r->k = (o && o->spec_k) ? o->spec_k : 4;
  r->k_cse = (o && o->spec_k) ? o->spec_k : 8;  // CSE: up to 8 lookback candidates per chunk
  r->L = (o && o->lookback) ? o->lookback : 2;
  r->qs_cap = (o && o->qs_cap) ? o->qs_cap : 16;
  r->vr_end = (o && o->vr_end) ? o->vr_end : 16;
  r->vr_oth = (o && o->vr_others) ? o->vr_others : 16;
  r->st = o ? reinterpret_cast<cudaStream_t>(o->stream) : nullptr;
  if (r->B % 16 != 0) return fail(FSM_EINVAL, "chunk_bytes must be a multiple of 16");
  if (r->k < 1 || r->k > kQsMax) return fail(FSM_EINVAL, "spec_k must be in [1,16]");
  if (r->L < 2 || r->L > kLookbackMax) return fail(FSM_EUNSUPPORTED, "lookback must be in [2,16] (P:300, R25)");
  if (r->qs_cap < 1 || r->qs_cap > kQsMax) return fail(FSM_EINVAL, "qs_cap must be in [1,16]");
  if (r->vr_end < 1 || r->vr_end > kVrMax || r->vr_oth < 1 || r->vr_oth > kVrMax)
    return fail(FSM_EINVAL, "vr_end / vr_others must be in [1,16]");
  if ((int)r->scheme < 0 || (int)r->scheme > FSM_SCHEME_PM_TREE) return fail(FSM_EINVAL, "unknown scheme");
  return FSM_OK;
}

// ---- scratch ------------------------------------------------------------------
int ensure_records(fsm_t f, uint64_t N) {
  if (f->rs_cap >= N && f->rs_base) return FSM_OK;
  if (f->rs_base) cudaFree(f->rs_base);
  f->rs_base = nullptr;
  f->rs_cap = 0;
  uint64_t cap = std::max<uint64_t>(N, 1024);
  cap = (cap + 255) & ~255ull;
  // carve the store: a dry run (base = null) sizes it, the second pass assigns pointers
  RecStore r{};
  auto carve = [&](uint8_t* base) -> uint64_t {
    uint64_t off = 0;
    auto take = [&](uint64_t bytes) -> uint8_t* {
      uint8_t* q = base ? base + off : nullptr;
      off += (bytes + 255) & ~255ull;
      return q;
    };
    r.cap = cap;
    r.start = (uint32_t*)take(4 * cap * kSlots);
    r.end = (uint32_t*)take(4 * cap * kSlots);
    r.cnt = (uint32_t*)take(4 * cap * kSlots);
    r.n_end = (uint32_t*)take(4 * cap);
    r.n_oth = (uint32_t*)take(4 * cap);
    r.oth_base = (uint32_t*)take(4 * cap);
    r.ref_start = (uint32_t*)take(4 * cap);
    r.ref_end = (uint32_t*)take(4 * cap);
    r.ref_cnt = (uint32_t*)take(4 * cap);
    r.x = (uint32_t*)take(4 * (cap + 8));
    r.cur_end = (uint32_t*)take(4 * cap);
    r.prefU = (uint32_t*)take(4 * cap);
    r.task_chunk = (uint32_t*)take(4 * (cap + 8));
    r.task_start = (uint32_t*)take(4 * (cap + 8));
    r.task_j = (uint32_t*)take(4 * (cap + 8));
    r.tstart = (uint32_t*)take(4 * (cap + 8));
    r.bflag = (uint32_t*)take(4 * (cap / 32 + 8) + 64);
    r.v0c = base ? reinterpret_cast<unsigned long long*>(r.bflag + cap / 32 + 8) : nullptr;
    r.next_qs = take(cap);
    r.found = take(cap);
    r.ulen = take(cap);
    r.upos = take(cap * kQsMax);
    r.next_new = take(cap);
    r.hcnt = take(cap);
    return off;
  };
  const uint64_t bytes = carve(nullptr);
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e != cudaSuccess) return fail(FSM_ENOMEM, std::string("record store: ") + cudaGetErrorString(e));
  carve(reinterpret_cast<uint8_t*>(p));
  e = cudaMemset(r.bflag, 0, 4 * (cap / 32 + 8) + 64);  // boundary counters start even (never reset), v0c zero
  if (e != cudaSuccess) return fail(FSM_ECUDA, std::string("record store: ") + cudaGetErrorString(e));
  f->rs = r;
  f->rs_base = p;
  f->rs_cap = cap;
  return FSM_OK;
}

int ensure_ctl(fsm_t f) {
  if (!f->d_ctl) CUDA_TRY(cudaMalloc(&f->d_ctl, sizeof(Ctl)));
  if (!f->h_ctl) {
    CUDA_TRY(cudaMallocHost(&f->h_ctl, sizeof(Ctl) * fsm_s::kRing));
    for (auto& slot : f->ev)
      for (auto& e : slot) CUDA_TRY(cudaEventCreate(&e));
  }
  const size_t need = 2 * 4096 + 64;
  if (f->block_tmp_elems < need) {
    if (f->d_block_tmp) cudaFree(f->d_block_tmp);
    CUDA_TRY(cudaMalloc(&f->d_block_tmp, need * sizeof(uint64_t)));
    f->block_tmp_elems = need;
  }
  return FSM_OK;
}

void fill_result_stats(fsm_result* out, const Ctl& h) {
  out->rounds = (uint32_t)h.rounds;
  out->tasks_mustdo = h.tasks_mustdo;
  out->tasks_sre = h.tasks_sre;
  out->tasks_helper = h.tasks_helper;
  out->tasks_total = h.tasks_mustdo + h.tasks_sre + h.tasks_helper;
  out->reread_bytes = h.reread_bytes;
  out->verify_checks = h.verify_checks;
  out->verify_matches = h.verify_matches;
  out->avg_active_workers = h.rounds ? (double)h.active_sum / (double)h.rounds : 0.0;
  out->pm_merge_checks = h.pm_merge_checks;
  out->pm_invalid_marks = h.pm_invalid_marks;
  out->pm_jumps = h.pm_jumps;
  out->helper_walks = h.helper_walks;
  out->task_walked_bytes = h.walked_bytes;
}

int select_auto(fsm_t f, const uint8_t* d_in, uint64_t len, const fsm_run_opts* opts);

// Lookback L > 2 (reading R25): the per-pair full images with multiplicities (built once,
// at the first such run) and the per-run table QS_c for every chunk (k_qs_long).
int prepare_long_lookback(fsm_t f, const uint8_t* d_in, uint64_t N, const Opts& o, RunParams* rp,
                          uint32_t* launches) {
  if (o.L <= 2) return FSM_OK;
  const uint32_t C = f->img.C, nt = f->n + 1;
  const uint64_t npairs = (uint64_t)C * C;
  if (!f->img2_base) {
    CUDA_TRY(cudaMalloc(&f->img2_base, npairs * kImgFull * 8 + npairs + 16));
    f->img2_s = reinterpret_cast<uint32_t*>(f->img2_base);
    f->img2_m = f->img2_s + npairs * kImgFull;
    f->img2_n = reinterpret_cast<uint8_t*>(f->img2_m + npairs * kImgFull);
    uint32_t grid = (uint32_t)std::min<uint64_t>(npairs, (uint64_t)f->sm_count * 4);
    if ((uint64_t)grid * nt > (1ull << 28)) grid = (uint32_t)std::max<uint64_t>(1, (1ull << 28) / nt);
    void* scratch = nullptr;
    CUDA_TRY(cudaMalloc(&scratch, (uint64_t)grid * nt * 4));
    cudaError_t ce = launch_build_img2_raw(f->d_ttc, f->n, C, (uint32_t*)scratch, grid, f->img2_s, f->img2_m,
                                           f->img2_n, o.st);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(o.st);
    cudaFree(scratch);
    CUDA_TRY(ce);
  }
  if (f->qsc_cap < N) {
    CUDA_TRY(cudaStreamSynchronize(o.st));  // queued runs may still read the old table
    if (f->qsc_base) cudaFree(f->qsc_base);
    f->qsc_base = nullptr;
    f->qsc_cap = 0;
    CUDA_TRY(cudaMalloc(&f->qsc_base, N * (kQsMax * 4 + 1) + 16));
    f->qsc_cap = N;
  }
  uint32_t* qsc = reinterpret_cast<uint32_t*>(f->qsc_base);
  uint8_t* qsl = reinterpret_cast<uint8_t*>(qsc + f->qsc_cap * kQsMax);
  CUDA_TRY(launch_qs_long(f->img, f->d_ttc, d_in, o.B, N, o.L, f->img2_s, f->img2_m, f->img2_n, qsc, qsl,
                          f->sm_count, o.st));
  rp->qsc = qsc;
  rp->qsc_len = qsl;
  *launches += 1;
  return FSM_OK;
}

// Enqueue one device run over d_in[0..len) from transformed start q0t on
// o.st; returns a ticket.  Everything (init, kernels, readback) is stream
// ordered, so runs on one handle may be queued back to back.
int run_enqueue(fsm_t f, const uint8_t* d_in, uint64_t len, const Opts& o, fsm_scheme scheme, uint32_t q0t,
                uint32_t* d_chunk_ends, uint64_t* ticket, const uint32_t* q0_dev = nullptr) {
  const uint64_t N = (len + o.B - 1) / o.B;
  int rc = ensure_ctl(f);
  if (rc) return rc;
  const uint64_t seq = f->next_seq++;
  const uint32_t slot = (uint32_t)(seq % fsm_s::kRing);
  auto& pd = f->pend[slot];
  if (pd.active) CUDA_TRY(cudaEventSynchronize(f->ev[slot][pd.done_ev]));  // ring wrapped: slot's readback must be done
  pd = fsm_s::Pending{seq, N, scheme, q0t, true};
  *ticket = seq;
  if (N == 0) return FSM_OK;
  RunParams rp{};
  rp.in = d_in;
  rp.q0t = q0t;
  rp.len = len;
  rp.B = o.B;
  rp.N = N;
  rp.scheme = scheme;
  rp.k = (scheme == FSM_SCHEME_PM || scheme == FSM_SCHEME_PM_TREE) ? o.k : scheme == FSM_SCHEME_CSE ? o.k_cse : 1;
  rp.qs_cap = o.qs_cap;
  rp.vr_end = o.vr_end;
  rp.vr_oth = o.vr_oth;
  rp.q0_dev = q0_dev;
  rp.stamps = stamps_enabled() ? 1u : 0u;
  rp.lazy_helpers = lazy_helpers_enabled() ? 1u : 0u;
  cudaEvent_t* ev = f->ev[slot];
  Ctl& h = f->h_ctl[slot];
  std::memset(&h, 0, sizeof(Ctl));
  h.f = 0;
  h.tf = q0t;
  h.fmin = N;
  h.it_fm[0] = N;  // first relaxation pass slot
  if ((scheme == FSM_SCHEME_ENUM || scheme == FSM_SCHEME_PM_TREE) && q0_dev)
    scheme = FSM_SCHEME_SRE;  // device-resident start: pipeline path
  if (scheme == FSM_SCHEME_ENUM) {
    if (f->n + 1 > kEnumMax) {
      pd.active = false;
      return fail(FSM_EUNSUPPORTED, "ENUM needs nstates + 1 <= 64");
    }
    // sub-chunk size E | B: small enough for parallelism, bounded scratch.  A stream of at
    // most enum_small_max_sub() sub-chunks of >= 64 B runs as ONE launch (k_enum_small)
    uint32_t Es = o.B;
    while (Es % 32 == 0 && Es > 64 && (len + Es / 2 - 1) / (Es / 2) <= enum_small_max_sub()) Es /= 2;
    // (only for short sub-chunks: 8192 threads walking long sub-chunks would be latency-bound;
    // longer streams keep the multi-level scan with many more threads)
    const bool small = len > 0 && Es <= 256 && (len + Es - 1) / Es <= enum_small_max_sub() &&
                       f->n + 1 <= kEnumSmallMax;
    const uint32_t E = small ? Es : enum_sub_bytes(o.B, len);
    const uint64_t nsub = (len + E - 1) / E;
    const uint64_t need = small ? enum_small_scratch_bytes(nsub) : enum_scratch_bytes(nsub);
    if (f->enum_bytes < need) {
      CUDA_TRY(cudaStreamSynchronize(o.st));  // earlier queued runs may still use the old scratch
      if (f->enum_base) cudaFree(f->enum_base);
      f->enum_base = nullptr;
      f->enum_bytes = 0;
      CUDA_TRY(cudaMalloc(&f->enum_base, need));
      f->enum_bytes = need;
    }
    rp.ctl_init = f->d_ctl;  // the walk kernel initialises the control block (no H2D copy)
    rp.h_out = &h;           // ... and the output kernel writes it back (pinned, UVA)
    if (small && !f->enum_ticket) {
      CUDA_TRY(cudaMalloc(&f->enum_ticket, 256));
      CUDA_TRY(cudaMemset(f->enum_ticket, 0, 256));
    }
    CUDA_TRY(cudaEventRecord(ev[0], o.st));
    NvtxRange nv_("enum (walk + composition scan)");
    if (small) {
      CUDA_TRY(launch_enum_small(f->img, rp, E, f->enum_base, f->enum_ticket, d_chunk_ends, f->d_ctl, o.st));
      pd.launches = 1;
    } else {
      CUDA_TRY(launch_enum_full(f->img, rp, E, f->enum_base, d_chunk_ends, f->d_ctl, &f->d_ctl->xfin, o.st,
                                f->sm_count));
      uint32_t L = 1;  // map levels: walk + L group scans + L descents + outputs
      for (uint64_t c = nsub; c > 64 && L < 16; c = (c + 63) / 64) L++;
      pd.launches = 2 + 2 * L;
    }
    CUDA_TRY(cudaEventRecord(ev[1], o.st));
    CUDA_TRY(cudaEventRecord(ev[2], o.st));
  } else if (scheme == FSM_SCHEME_PM_TREE) {
    // faithful PM (pm_tree.cu): spec-k round 0, tree merge rounds, sequential stage 2, descent
    if (f->rs_cap < N) CUDA_TRY(cudaStreamSynchronize(o.st));
    if ((rc = ensure_records(f, N))) return rc;
    const size_t need = pm_tree_scratch_bytes(N, o.k, nullptr);
    if (f->pm_bytes < need) {
      CUDA_TRY(cudaStreamSynchronize(o.st));
      if (f->pm_base) cudaFree(f->pm_base);
      f->pm_base = nullptr;
      f->pm_bytes = 0;
      CUDA_TRY(cudaMalloc(&f->pm_base, need));
      f->pm_bytes = need;
    }
    rp.ctl_init = f->d_ctl;
    CUDA_TRY(cudaEventRecord(ev[0], o.st));
    uint32_t lq = 0;
    if ((rc = prepare_long_lookback(f, d_in, N, o, &rp, &lq))) return rc;
    {
      NvtxRange nv_("speculative execution spec-k (PM round 0)");
      CUDA_TRY(launch_spec_exec(f->img, rp, f->rs, o.st));
    }
    pd.launches = lq + 1 + (len % o.B != 0 && len / o.B > 0);
    rp.ctl_init = nullptr;
    CUDA_TRY(cudaEventRecord(ev[1], o.st));
    uint32_t nl = 0;
    {
      NvtxRange nv_("PM tree merge + sequential stage 2");
      CUDA_TRY(launch_pm_tree(f->img, rp, f->rs, o.k, f->pm_base, f->d_ctl, d_chunk_ends, f->sm_count, o.st, &nl));
    }
    pd.launches += nl;
    CUDA_TRY(cudaEventRecord(ev[2], o.st));
  } else {
    if (f->rs_cap < N) CUDA_TRY(cudaStreamSynchronize(o.st));  // growing the store: drain queued runs
    if ((rc = ensure_records(f, N))) return rc;
    rp.ctl_init = f->d_ctl;  // the spec kernel initialises the control block
    rp.h_out = &h;           // ... and the verify kernel's finalize step writes it back (pinned, UVA)
    CUDA_TRY(cudaEventRecord(ev[0], o.st));
    uint32_t lq = 0;
    if ((rc = prepare_long_lookback(f, d_in, N, o, &rp, &lq))) return rc;
    // dense recovery rounds go to the TMA task kernel (SRE / RR / NF on low-accuracy DFAs); this
    // needs a host check per verify launch, so it is off when the profile says the
    // speculation is accurate (no dense rounds expected)
    rp.dense = ((scheme == FSM_SCHEME_SRE || scheme == FSM_SCHEME_CSE || scheme == FSM_SCHEME_RR ||
                 scheme == FSM_SCHEME_NF) && len / o.B > 0 && o.B % 64 == 0 &&
                (reinterpret_cast<uintptr_t>(d_in) & 15u) == 0 && f->acc1_hint < 0.5) ? 1u : 0u;
    // R30: the round-0 TMA walk checkpoints its path so dense tasks stop where they meet it
    {
      const uint32_t sh = ck_shift_default();
      if (rp.dense && rp.k == 1 && sh && !spec_path_generic_only() && o.B % (1u << sh) == 0 &&
          o.B >= (2u << sh) && f->conv_hint > 0.0) {
        const size_t nck = (size_t)(o.B / (1u << sh) - 1) * N * sizeof(uint2);
        const size_t need = ((nck + 255) & ~(size_t)255) + 2 * f->rs.cap * 16;  // + the passes' chain lists
        if (f->ck_bytes < need) {
          CUDA_TRY(cudaStreamSynchronize(o.st));  // queued runs may still read the old array
          if (f->ck_base) cudaFree(f->ck_base);
          f->ck_base = nullptr;
          f->ck_bytes = 0;
          CUDA_TRY(cudaMalloc(&f->ck_base, need));
          f->ck_bytes = need;
        }
        rp.ck = reinterpret_cast<uint2*>(f->ck_base);
        rp.ck_shift = sh;
        rp.ck_seg = ck_seg_for(o.B, sh);
        rp.ck_list = reinterpret_cast<uint8_t*>(f->ck_base) + ((nck + 255) & ~(size_t)255);
      }
    }
    {
      // accurate SRE (no dense rounds expected): round 0's verification and its inline
      // recoveries run inside the TMA spec kernel as its tiles finish (RunParams::v0); the
      // verify launch then returns at once unless a recovery moved an end
      const bool tma_full = !spec_path_generic_only() && len % o.B == 0 && len / o.B > 0 && o.B % 64 == 0 &&
                            (reinterpret_cast<uintptr_t>(d_in) & 15u) == 0 && len / o.B < (1ull << 31);
      rp.v0 = (scheme == FSM_SCHEME_SRE && rp.k == 1 && !rp.dense && tma_full && !v0_disabled()) ? 1u : 0u;
      rp.v0_ctl = f->d_ctl;
      rp.v0_bflag = f->rs.bflag;
      rp.v0_chunk_ends = d_chunk_ends;
      rp.tma_evict_normal = tma_evict_mode() == 1 ? 1u : 0u;
      NvtxRange nv_("speculative execution (round 0)");
      uint64_t tma_done = 0;
      CUDA_TRY(launch_spec_exec(f->img, rp, f->rs, o.st, &tma_done));
      if (tma_done < len / o.B) rp.ck_shift = 0;  // the full chunks were not walked by the TMA kernel: no checkpoints
    }
    {  // TMA kernel over the full chunks + the generic kernel for a tail chunk (or everything)
      const bool tma = !spec_path_generic_only() && len / o.B > 0 && o.B % 64 == 0 &&
                       (reinterpret_cast<uintptr_t>(d_in) & 15u) == 0;
      pd.launches = lq + (tma ? 1 + (len % o.B != 0) : 1);
    }
    rp.ctl_init = nullptr;  // initialised by the spec kernel; later launches must not touch it
    CUDA_TRY(cudaEventRecord(ev[1], o.st));
    // dense rounds are device-driven: `slots` (task kernel + finish + verify) triples are
    // queued behind the first verify launch; a verify launch that needs a dense round
    // hands it to the next triple, or runs it in-kernel when none is left; launches after
    // the run completed return at once.  No host round trip: runs stay queued back to back.
    const uint32_t slots = rp.dense ? f->dense_hint : 0;
    rp.dense_slots = slots;
    NvtxRange nv_("verification + recovery (+ dense-round slots)");
    CUDA_TRY(launch_verify_recover(f->img, rp, f->rs, f->d_ctl, f->d_block_tmp, d_chunk_ends, o.st, f->sm_count));
    pd.launches++;
    for (uint32_t r = 0; r < slots; r++) {
      CUDA_TRY(launch_task_dense(f->img, rp, f->rs, f->d_ctl, f->sm_count, o.st));
      rp.dense_slots = slots - 1 - r;
      CUDA_TRY(launch_verify_recover(f->img, rp, f->rs, f->d_ctl, f->d_block_tmp, d_chunk_ends, o.st, f->sm_count));
      // task kernel (R30: one launch per segment pass) + finish + verify (no-ops once the run is complete)
      const bool seg = rp.ck_shift && rp.ck_seg;  // (no tail chunk: the last pass commits, no finish kernel)
      pd.launches += (seg && len % o.B == 0 ? 1u : 2u) + (seg ? (o.B + rp.ck_seg - 1) / rp.ck_seg : 1u);
    }
    pd.dense_slots = slots;
    pd.dense = rp.dense != 0;
    CUDA_TRY(cudaEventRecord(ev[2], o.st));
  }
  if (rp.h_out) {
    pd.done_ev = 2;  // the verify kernel wrote the result to the pinned slot
  } else {
    CUDA_TRY(cudaMemcpyAsync(&h, f->d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, o.st));
    CUDA_TRY(cudaEventRecord(ev[3], o.st));
  }
  return FSM_OK;
}

// Wait for a ticket and fill the result (transformed final state in *final_tid).
int run_collect(fsm_t f, uint64_t ticket, fsm_result* out, uint32_t* final_tid) {
  const uint32_t slot = (uint32_t)(ticket % fsm_s::kRing);
  auto& pd = f->pend[slot];
  if (!pd.active || pd.seq != ticket) return fail(FSM_EINVAL, "unknown or already collected ticket");
  std::memset(out, 0, sizeof(*out));
  out->nchunks = pd.N;
  out->scheme_used = pd.scheme;
  pd.active = false;
  if (pd.N == 0) {
    *final_tid = pd.q0t;
    return FSM_OK;
  }
  CUDA_TRY(cudaEventSynchronize(f->ev[slot][pd.done_ev]));
  const Ctl& h = f->h_ctl[slot];
  float t1 = 0, t2 = 0;
  cudaEventElapsedTime(&t1, f->ev[slot][0], f->ev[slot][1]);
  cudaEventElapsedTime(&t2, f->ev[slot][1], f->ev[slot][2]);
  fill_result_stats(out, h);
  if (pd.dense) {  // size the next run's dense slots to the rounds this one used (0: none queued;
                   // a run that then needs one runs it in-kernel and sets dense_denied)
    const uint32_t used = h.dense_rounds + (h.dense_denied ? 1u : 0u);
    f->dense_hint = std::min<uint32_t>(16u, used);
  }
  f->last_nstamp = std::min<uint32_t>(h.nstamp, 24);
  std::copy(h.stamp, h.stamp + 24, f->last_stamp);
  std::copy(h.tl, h.tl + 4, f->last_tl);
  out->accept_count = h.accept_count;
  out->ms_spec = t1;
  out->ms_verify = t2;
  out->kernel_launches = pd.launches;
  *final_tid = h.xfin;
  return FSM_OK;
}

int run_core(fsm_t f, const uint8_t* d_in, uint64_t len, const Opts& o, fsm_scheme scheme, uint32_t q0t,
             uint32_t* d_chunk_ends, fsm_result* out, uint32_t* final_tid) {
  uint64_t t = 0;
  int rc = run_enqueue(f, d_in, len, o, scheme, q0t, d_chunk_ends, &t);
  if (rc) return rc;
  return run_collect(f, t, out, final_tid);
}

// Delta rows for MODE_U16D: a cold row of the transformed table
// is stored as (hot base row, <= kDeltaExc exception classes) when it differs from
// some hot row in that few columns — the rows of a literal/regex DFA's deep states
// are their failure state's row plus a goto or two.  Picks the hot-row count H
// that keeps the most frequency mass on chip within the smem budget
// (hot rows C*2 B each + 8 B per delta row); used only when every cold real
// row compresses.  The poison row (all poison) is stored once as hot row H.
// Output: the shared-memory image [hot rows 0..H-1][poison row][pad][delta rows].
bool plan_delta_rows(fsm_t f, const std::vector<uint32_t>& ttc, uint32_t nt, uint32_t C,
                     std::vector<uint32_t>& tid2code, std::vector<uint32_t>& code2tid, uint32_t budget_in,
                     DevImage* img, std::vector<uint2>* out) {
  const uint32_t budget = budget_in ? budget_in : 128 * 1024;
  const uint64_t row_b = (uint64_t)C * 2;
  const uint32_t nr = nt - 1;  // real states (the poison tid nr is handled apart)
  if (nr < 2 || row_b <= 8 || 2 * C > 254 || (uint64_t)nr * 8 + 2 * row_b + 512 > budget) return false;
  uint64_t hmax = (budget - (uint64_t)nr * 8 - row_b - 512) / (row_b - 8);  // (H+1)*row + (nr-H)*8 <= budget
  hmax = std::min<uint64_t>(hmax, nr - 1);
  // pre-multiplied codes: (H+1)*C + cold tids < 2^15, hot byte offsets + the smem base < 2^16
  while (hmax >= 1 && ((hmax + 1) * C + (nr - hmax) > 0x7FFFu || 2 * (hmax + 1) * C + kDeltaBaseMax > 0xFFFFu))
    hmax--;
  if (hmax < 1) return false;
  // first[t][d] = smallest j < min(t, hmax) whose row differs from row t in <= d columns
  const uint32_t kNo = 0xFFFFFFFFu;
  std::vector<uint32_t> first((uint64_t)nr * (kDeltaExc + 1), kNo);
  for (uint32_t t = 1; t < nr; t++) {
    const uint32_t* rt = &ttc[(uint64_t)t * C];
    uint32_t* ft = &first[(uint64_t)t * (kDeltaExc + 1)];
    const uint32_t jm = (uint32_t)std::min<uint64_t>(t, hmax);
    for (uint32_t j = 0; j < jm && ft[0] == kNo; j++) {
      const uint32_t* rj = &ttc[(uint64_t)j * C];
      uint32_t d = 0;
      for (uint32_t c = 0; c < C && d <= kDeltaExc; c++) d += rt[c] != rj[c];
      for (uint32_t e = d; e <= kDeltaExc; e++)
        if (ft[e] == kNo) ft[e] = j;
    }
  }
  // smallest H with every real row hot or compressible (more room for TMA stages)
  uint64_t H = 0;
  for (uint64_t h = 1; h <= hmax && !H; h++) {
    bool ok = true;
    for (uint64_t t = h; t < nr && ok; t++) ok = first[t * (kDeltaExc + 1) + kDeltaExc] < h;
    if (ok) H = h;
  }
  if (!H) return false;
  if (const char* e = getenv("GSPEC_DELTA_H")) {  // experiments: a larger hot set (fewer delta lookups)
    const uint64_t want = strtoull(e, nullptr, 10);
    if (want > H) H = std::min<uint64_t>(want, hmax);
  }
  // One-exception plan (the step drops a compare and a select): the smallest H1 >= H such that
  // the rows needing two exceptions against [0, H1) — X — can be hot too (slots H1+1..), within
  // the budget and the code limits.  GSPEC_DELTA_EXC=2 keeps the two-exception plan (A/B).
  std::vector<uint32_t> X;
  uint32_t exc = kDeltaExc;
  {
    const char* e = getenv("GSPEC_DELTA_EXC");
    if (!(e && atoi(e) == 2)) {
      for (uint64_t h1 = H; h1 <= hmax; h1++) {
        std::vector<uint32_t> x;
        bool ok = true;
        for (uint64_t t = h1; t < nr && ok; t++) {
          const uint32_t* ft = &first[t * (kDeltaExc + 1)];
          if (!(ft[0] < h1 || ft[1] < h1)) x.push_back((uint32_t)t);
          ok = h1 + x.size() <= hmax;
        }
        const uint64_t hot = h1 + 1 + x.size(), ncold = nr - h1 - x.size();
        if (!ok || hot * C + ncold > 0x7FFFu || 2 * hot * C + kDeltaBaseMax > 0xFFFFu) continue;
        const uint64_t bytes1 = ((hot * C * 2 + 255) & ~255ull) + 256 + ncold * 8;
        if (bytes1 > budget) continue;
        H = h1;
        X = std::move(x);
        exc = 1;
        break;
      }
    }
  }
  // codes: hot t -> slot*C (top-H tids: slot t; poison: slot H, stored as hot row H; the X tids:
  // slots H+1..), cold t -> HC1 + its rank among the cold tids
  const uint64_t HC1 = (H + 1 + X.size()) * C;
  std::vector<uint32_t> slot(nt, 0xFFFFFFFFu);
  for (uint32_t t = 0; t < H; t++) slot[t] = t;
  slot[nr] = (uint32_t)H;
  for (size_t i = 0; i < X.size(); i++) slot[X[i]] = (uint32_t)(H + 1 + i);
  std::vector<uint32_t> code(nt), cold;
  for (uint32_t t = 0; t < nt; t++) {
    const uint32_t a = tid2code[t] >> 15;  // accept flag of the plain u16 code
    uint64_t c;
    if (slot[t] != 0xFFFFFFFFu) {
      c = (uint64_t)slot[t] * C;
    } else {
      c = HC1 + cold.size();
      cold.push_back(t);
    }
    code[t] = (uint32_t)c | (a << 15);
  }
  const uint64_t hot_b = HC1 * 2;
  const uint64_t cls_off = (hot_b + 255) & ~255ull;
  const uint64_t delta_off = cls_off + 256;
  const uint64_t bytes = (delta_off + (uint64_t)cold.size() * 8 + 15) & ~15ull;
  if (bytes > budget) return false;
  std::vector<uint16_t> im(bytes / 2, 0);
  for (uint64_t t = 0; t < H; t++)
    for (uint32_t c = 0; c < C; c++) im[t * C + c] = (uint16_t)code[ttc[t * C + c]];
  for (uint32_t c = 0; c < C; c++) im[H * C + c] = (uint16_t)code[nr];
  for (size_t i = 0; i < X.size(); i++)
    for (uint32_t c = 0; c < C; c++) im[(H + 1 + i) * C + c] = (uint16_t)code[ttc[(uint64_t)X[i] * C + c]];
  uint8_t* cm = reinterpret_cast<uint8_t*>(im.data()) + cls_off;
  for (uint32_t b = 0; b < 256; b++) cm[b] = (uint8_t)(2 * f->cls[b]);
  uint2* dl = reinterpret_cast<uint2*>(reinterpret_cast<uint8_t*>(im.data()) + delta_off);
  for (size_t ci = 0; ci < cold.size(); ci++) {
    const uint32_t t = cold[ci];
    const uint32_t* ft = &first[(uint64_t)t * (kDeltaExc + 1)];
    uint32_t j = kNo;
    for (uint32_t e = 0; e <= exc && j == kNo; e++)
      if (ft[e] < H) j = ft[e];
    if (j == kNo) return false;  // unreachable (checked above)
    uint32_t ex[kDeltaExc] = {0xFF, 0xFF}, ec[kDeltaExc] = {0, 0}, k = 0;
    for (uint32_t c = 0; c < C; c++)
      if (ttc[(uint64_t)t * C + c] != ttc[(uint64_t)j * C + c]) {
        ex[k] = 2 * c;
        ec[k] = code[ttc[(uint64_t)t * C + c]];
        k++;
      }
    dl[ci] = make_uint2((uint32_t)(2 * C * j) << 16 | ex[1] << 8 | ex[0], (ec[0] & 0xFFFFu) | (ec[1] << 16));
  }
  out->assign(reinterpret_cast<const uint2*>(im.data()), reinterpret_cast<const uint2*>(im.data()) + bytes / 8);
  tid2code = code;
  code2tid.assign(0x8000, nr);
  for (uint32_t t = 0; t < nt; t++) code2tid[code[t] & 0x7FFFu] = t;
  img->H = (uint32_t)H;
  img->D = (uint32_t)cold.size();
  img->delta_exc = exc;
  img->HC1 = (uint32_t)HC1;
  img->cls_off = (uint32_t)cls_off;
  img->delta_off = (uint32_t)delta_off;
  img->smem_table_bytes = (uint32_t)bytes;
  return true;
}

fsm_scheme tree_select(const fsm_features& ft, uint32_t n) {
  // Fig. 6 (image lost) reconstructed from P:284-290, P:339-345, P:383 (R19)
  if (n <= 63 && ft.uniq10 >= n / 2.0) return FSM_SCHEME_ENUM;  // n + poison <= 64 map entries
  if (ft.uniq10 <= 4.0) return FSM_SCHEME_SRE;
  if (ft.acck >= 0.9 && ft.acck - ft.acc1 >= 0.2) return FSM_SCHEME_PM;
  // R19b: helpers cost a full chunk walk on a saturated GPU; RR/NF only when the
  // extra lookback candidates catch most mispredictions (GSPEC_SELECTOR=paper: the
  // reconstructed tree without this gate)
  const char* sel = getenv("GSPEC_SELECTOR");
  const bool paper = sel && std::strcmp(sel, "paper") == 0;
  if (!paper && ft.acck - ft.acc1 < 0.5) return FSM_SCHEME_SRE;
  if (ft.input_sensitivity >= 0.2) return FSM_SCHEME_NF;
  return FSM_SCHEME_RR;
}

}  // namespace

extern "C" {

int gspec_set_error(int code, const char* msg) { return fail(code, msg); }

const char* fsm_last_error(void) { return g_err.c_str(); }

const char* fsm_strerror(int s) {
  switch (s) {
    case FSM_OK: return "ok";
    case FSM_EINVAL: return "invalid argument";
    case FSM_ENOMEM: return "out of memory";
    case FSM_ECUDA: return "CUDA error";
    case FSM_EAGAIN: return "retry (speculative shard map invalid)";
    case FSM_ESYMBOL: return "input symbol out of range";
    case FSM_ENCCL: return "collective failed";
    case FSM_EUNSUPPORTED: return "unsupported";
    default: return "unknown status";
  }
}

uint64_t fsm_num_chunks(uint64_t len, uint32_t chunk_bytes) {
  if (!chunk_bytes) chunk_bytes = 4096;
  return (len + chunk_bytes - 1) / chunk_bytes;
}

int fsm_load(const uint32_t* table, uint32_t n, uint32_t nsyms, uint32_t start, const uint8_t* accept,
             const fsm_load_opts* opts, fsm_t* out) {
  ApiScope api_scope_("fsm_load");
  if (!table || !accept || !out) return fail(FSM_EINVAL, "NULL table/accept/out");
  if (n == 0 || nsyms == 0 || nsyms > 256 || start >= n) return fail(FSM_EINVAL, "bad nstates/nsyms/start");
  if (n >= (1u << 24)) return fail(FSM_EUNSUPPORTED, "nstates >= 2^24");
  for (uint64_t i = 0; i < (uint64_t)n * nsyms; i++)
    if (table[i] >= n) return fail(FSM_EINVAL, "table entry >= nstates");
  const uint32_t policy = opts ? opts->freq_policy : 0;
  if (policy > 1) return fail(FSM_EINVAL, "freq_policy must be 0 or 1");
  if (policy == 1 && (!opts->profile_sample || !opts->profile_len))
    return fail(FSM_EINVAL, "PROFILE policy needs a sample");
  fsm_t f = new fsm_s();
  f->n = n;
  f->nsyms = nsyms;
  f->q0 = start;
  f->table.assign(table, table + (uint64_t)n * nsyms);
  f->accept.assign(accept, accept + n);
  for (auto& a : f->accept) a = a ? 1 : 0;
  cudaGetDevice(&f->device);
  cudaDeviceGetAttribute(&f->sm_count, cudaDevAttrMultiProcessorCount, f->device);
  int rc = FSM_OK;
  auto bail = [&](int code) {
    fsm_free(f);
    return code;
  };

  // ---- 1. frequency-based transformation ----
  const uint32_t nt = n + 1, P = n;  // poison state: absorbing, ranked last
  f->freq.assign(n, 0);
  if (policy == 0) {
    for (uint64_t i = 0; i < (uint64_t)n * nsyms; i++) f->freq[table[i]]++;  // static in-degree
  } else {
    uint32_t s = start;
    f->freq[s]++;
    for (uint64_t i = 0; i < opts->profile_len; i++) {
      const uint8_t b = opts->profile_sample[i];
      if (b >= nsyms) break;
      s = table[(uint64_t)s * nsyms + b];
      f->freq[s]++;
    }
  }
  std::vector<uint32_t> order(n);
  std::iota(order.begin(), order.end(), 0u);
  std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return f->freq[a] > f->freq[b]; });
  f->perm.assign(nt, 0);
  f->inv.assign(nt, 0);
  for (uint32_t r = 0; r < n; r++) {
    f->inv[r] = order[r];
    f->perm[order[r]] = r;
  }
  f->perm[P] = P;
  f->inv[P] = P;
  std::vector<uint8_t> acc_t(nt, 0);
  for (uint32_t t = 0; t < n; t++) acc_t[t] = f->accept[f->inv[t]];

  // ---- 2. byte classes: identical columns; bytes >= nsyms -> poison class ----
  f->cls.assign(256, 0);
  std::map<std::vector<uint32_t>, uint32_t> colmap;
  std::vector<uint32_t> rep;  // representative byte of each class
  for (uint32_t b = 0; b < nsyms; b++) {
    std::vector<uint32_t> col(n);
    for (uint32_t q = 0; q < n; q++) col[q] = table[(uint64_t)q * nsyms + b];
    auto it = colmap.find(col);
    if (it == colmap.end()) {
      const uint32_t id = (uint32_t)rep.size();
      colmap.emplace(std::move(col), id);
      rep.push_back(b);
      f->cls[b] = (uint8_t)id;
    } else {
      f->cls[b] = (uint8_t)it->second;
    }
  }
  uint32_t C = (uint32_t)rep.size();
  const bool has_poison_cls = nsyms < 256;
  const uint32_t PC = C;
  if (has_poison_cls) {
    for (uint32_t b = nsyms; b < 256; b++) f->cls[b] = (uint8_t)PC;
    C++;
  }
  if (C > 256) return bail(fail(FSM_EINVAL, "too many classes"));
  // transformed tid x class table
  std::vector<uint32_t> ttc((uint64_t)nt * C);
  for (uint32_t t = 0; t < nt; t++)
    for (uint32_t c = 0; c < C; c++) {
      uint32_t v;
      if (t == P || (has_poison_cls && c == PC)) v = P;
      else v = f->perm[table[(uint64_t)f->inv[t] * nsyms + rep[c]]];
      ttc[(uint64_t)t * C + c] = v;
    }

  // ---- 3. table format and codes ----
  uint32_t n_acc = 0;
  for (uint32_t t = 0; t < nt; t++) n_acc += acc_t[t];
  const uint32_t n_na = nt - n_acc;
  uint32_t force = opts ? opts->force_mode : 0;
  if (force > 4) return bail(fail(FSM_EINVAL, "force_mode must be 0..4"));
  const bool want_delta = force == 0 || force == 4;  // 4: u16 classed with delta rows
  if (force == 4) force = MODE_U16;
  uint32_t mode;
  if (force) mode = force;
  else if (n_na <= 128 && n_acc <= 128) mode = MODE_U8;
  else if (nt <= 32768) mode = MODE_U16;
  else mode = MODE_U32;
  if (mode == MODE_U8 && !(n_na <= 128 && n_acc <= 128)) return bail(fail(FSM_EUNSUPPORTED, "u8 mode needs <=128 accepting and non-accepting states"));
  if (mode == MODE_U16 && nt > 32768) return bail(fail(FSM_EUNSUPPORTED, "u16 mode needs nstates < 32768"));
  if (mode < MODE_U8 || mode > MODE_U32) return bail(fail(FSM_EINVAL, "force_mode must be 0..3"));
  DevImage& img = f->img;
  img.mode = mode;
  img.n = n;
  img.nsyms = nsyms;
  img.C = C;
  img.q0t = f->perm[start];
  std::vector<uint32_t> tid2code(nt), code2tid(256, P);
  if (mode == MODE_U8) {
    uint32_t max_code = 0;
    if (opts && opts->profile_sample && opts->profile_len) {
      place_rows_bank_aware(f, ttc, C, acc_t, n_na, n_acc, opts->profile_sample, opts->profile_len, tid2code,
                            code2tid);
    } else {
      uint32_t na = 0, ac = 0;
      for (uint32_t t = 0; t < nt; t++) {
        const uint32_t code = acc_t[t] ? 128 + ac++ : na++;
        tid2code[t] = code;
        code2tid[code] = t;
      }
    }
    for (uint32_t t = 0; t < nt; t++) max_code = std::max(max_code, tid2code[t]);
    const uint32_t R = kRow8Bytes;  // row stride (walk.cuh kRow8): 4-byte pad rotates rows across banks
    std::vector<uint8_t> T8(256 * R, (uint8_t)tid2code[P]);
    for (uint32_t code = 0; code < 256; code++) {
      const uint32_t t = code2tid[code];
      for (uint32_t b = 0; b < 256; b++) T8[code * R + b] = (uint8_t)tid2code[ttc[(uint64_t)t * C + f->cls[b]]];
    }
    img.H = nt;
    img.smem_table_bytes = (((max_code + 1) * R) + 15) & ~15u;
    if ((rc = upload(f, &img.T8, T8))) return bail(rc);
  } else {
    const uint32_t shift = mode == MODE_U16 ? 15 : 31;
    for (uint32_t t = 0; t < nt; t++) tid2code[t] = t | ((uint32_t)acc_t[t] << shift);
    const uint32_t esz = mode == MODE_U16 ? 2 : 4;
    const uint32_t budget = (opts && opts->smem_budget_bytes) ? opts->smem_budget_bytes : 96 * 1024;
    uint64_t H = budget / (C * esz);
    if (H > nt) H = nt;
    img.H = (uint32_t)H;
    img.smem_table_bytes = (uint32_t)(((H * C * esz) + 15) & ~15ull);
    if (mode == MODE_U16 && H == nt && (uint64_t)nt * C <= 0x7FFFu && C < 128) {
      // every row hot: no hot test, and pre-multiplied codes (code = 2*t*C = the row's byte
      // offset, accept flag in bit 0; the staged class map holds 2*class), so a step is
      // LOP3 + IADD3 on the dependent chain instead of LOP3 + IMAD + IADD3
      img.mode = MODE_U16H;
      code2tid.assign(0x8000, P);
      for (uint32_t t = 0; t < nt; t++) {
        tid2code[t] = 2 * t * C | (uint32_t)acc_t[t];  // row byte offset | accept flag (bit 0)
        code2tid[t * C] = t;
      }
      std::vector<uint8_t> cls2(256);
      for (uint32_t b = 0; b < 256; b++) cls2[b] = (uint8_t)(2 * f->cls[b]);
      if ((rc = upload(f, &img.cls2, cls2))) return bail(rc);
    }
    std::vector<uint2> delta;
    if (mode == MODE_U16 && H < nt && want_delta && C < 128 &&
        plan_delta_rows(f, ttc, nt, C, tid2code, code2tid, opts ? opts->smem_budget_bytes : 0, &img, &delta)) {
      img.mode = MODE_U16D;
      if ((rc = upload(f, &img.Dl, delta))) return bail(rc);
    }
    if (mode == MODE_U16) {
      std::vector<uint16_t> T16((uint64_t)nt * C);
      for (uint64_t i = 0; i < T16.size(); i++) T16[i] = (uint16_t)tid2code[ttc[i]];
      if ((rc = upload(f, &img.T16, T16, 64))) return bail(rc);
    } else {
      std::vector<uint32_t> T32((uint64_t)nt * C);
      for (uint64_t i = 0; i < T32.size(); i++) T32[i] = tid2code[ttc[i]];
      if ((rc = upload(f, &img.T32, T32, 64))) return bail(rc);
    }
  }
  std::vector<uint32_t> inv_v(f->inv.begin(), f->inv.end());
  if ((rc = upload(f, &img.cls, f->cls))) return bail(rc);
  if ((rc = upload(f, &img.tid2code, tid2code))) return bail(rc);
  if ((rc = upload(f, &img.code2tid, code2tid))) return bail(rc);
  if ((rc = upload(f, &img.inv, inv_v))) return bail(rc);
  if ((rc = upload(f, &img.acc, acc_t))) return bail(rc);
  const uint32_t* d_ttc = nullptr;
  if ((rc = upload(f, &d_ttc, ttc))) return bail(rc);
  f->d_ttc = d_ttc;
  // multi-symbol step table for the enumerative walk on small alphabets: the
  // transformation P:319-330 applied to strings of K symbols — entry (tid, combo) is the tid
  // after the K symbols (a value >= nsyms -> poison) and how many of the K states accept
  img.TK = nullptr;
  img.tk_bytes = 0;
  img.tk_syms = 0;
  img.pk_off = 0;
  if (mode == MODE_U8 && nsyms <= 4 && nt <= 64) {
    const uint32_t K = nsyms <= 2 ? 8 : 4, bits = 8 / K, row = 257;  // words per row (kTkRow)
    const bool pk = K == 8 && nt <= 8 && !tk_pk_disabled();
    const uint64_t tk_words = ((uint64_t)nt * row + 3) & ~3ull;      // staged in 16-byte pieces
    std::vector<uint32_t> tk(tk_words + (pk ? 512 : 0), 0);
    for (uint32_t t = 0; t < nt; t++)
      for (uint32_t cb = 0; cb < 256; cb++) {
        uint32_t x = t, k = 0;
        for (uint32_t i = 0; i < K; i++) {
          const uint32_t sym = (cb >> (bits * i)) & ((1u << bits) - 1u);
          x = (x == P || sym >= nsyms) ? P : ttc[(uint64_t)x * C + f->cls[sym]];
          k += acc_t[x];
        }
        tk[(uint64_t)t * row + cb] = x * row * 4 | k << 24;
        if (pk)  // packed map: byte t of PK[cb] = next tid | count << 4 (tids and counts < 16)
          reinterpret_cast<uint8_t*>(tk.data() + tk_words)[cb * 8 + t] = (uint8_t)(x | k << 4);
      }
    if (pk) {
      for (uint32_t cb = 0; cb < 256; cb++)  // unused entries t >= nt: identity, no count
        for (uint32_t t = nt; t < 8; t++) reinterpret_cast<uint8_t*>(tk.data() + tk_words)[cb * 8 + t] = (uint8_t)t;
      img.pk_off = (uint32_t)(tk_words * 4);
    }
    if ((rc = upload(f, &img.TK, tk))) return bail(rc);
    img.tk_bytes = (uint32_t)tk.size() * 4;
    img.tk_syms = K;
  }

  // ---- 4. lookback pair table on the device ----
  const uint64_t npairs = (uint64_t)C * C;
  void *qs2 = nullptr, *qs2l = nullptr, *qs2i = nullptr, *scratch = nullptr;
  if ((rc = dev_alloc(f, &qs2, npairs * kQsMax * 4))) return bail(rc);
  if ((rc = dev_alloc(f, &qs2l, npairs + 16))) return bail(rc);
  if ((rc = dev_alloc(f, &qs2i, npairs * 4))) return bail(rc);
  uint32_t grid = (uint32_t)std::min<uint64_t>(npairs, (uint64_t)f->sm_count * 4);
  if ((uint64_t)grid * nt > (1ull << 28)) grid = (uint32_t)std::max<uint64_t>(1, (1ull << 28) / nt);
  cudaError_t ce = cudaMalloc(&scratch, (uint64_t)grid * nt * 4);
  if (ce != cudaSuccess) return bail(fail(FSM_ENOMEM, "qs2 scratch"));
  ce = launch_build_qs2_raw(d_ttc, n, C, (uint32_t*)scratch, grid, (uint32_t*)qs2, (uint8_t*)qs2l, (uint32_t*)qs2i, 0);
  if (ce == cudaSuccess) ce = cudaDeviceSynchronize();
  cudaFree(scratch);
  if (ce != cudaSuccess) return bail(fail(FSM_ECUDA, std::string("qs2 build: ") + cudaGetErrorString(ce)));
  img.qs2 = (const uint32_t*)qs2;
  img.qs2_len = (const uint8_t*)qs2l;
  img.qs2_img = (const uint32_t*)qs2i;
  *out = f;
  return FSM_OK;
}

void fsm_free(fsm_t f) {
  if (!f) return;
  for (void* p : f->owned) cudaFree(p);
  if (f->rs_base) cudaFree(f->rs_base);
  if (f->d_ctl) cudaFree(f->d_ctl);
  if (f->h_ctl) cudaFreeHost(f->h_ctl);
  for (auto& slot : f->ev)
    for (auto& e : slot)
      if (e) cudaEventDestroy(e);
  if (f->d_block_tmp) cudaFree(f->d_block_tmp);
  if (f->enum_base) cudaFree(f->enum_base);
  if (f->enum_ticket) cudaFree(f->enum_ticket);
  if (f->feat_base) cudaFree(f->feat_base);
  if (f->h_dev_in) cudaFree(f->h_dev_in);
  if (f->h_dev_ce) cudaFree(f->h_dev_ce);
  if (f->d_small) cudaFree(f->d_small);
  if (f->shard_base) cudaFree(f->shard_base);
  if (f->batch_base) cudaFree(f->batch_base);
  for (auto& e : f->batch_ev)
    if (e) cudaEventDestroy(e);
  if (f->multi_base) cudaFree(f->multi_base);
  if (f->pm_base) cudaFree(f->pm_base);
  if (f->ck_base) cudaFree(f->ck_base);
  if (f->prof_buf) cudaFree(f->prof_buf);
  if (f->img2_base) cudaFree(f->img2_base);
  if (f->qsc_base) cudaFree(f->qsc_base);
  if (f->h_sh) cudaFreeHost(f->h_sh);
  for (auto& e : f->sh_ev)
    if (e) cudaEventDestroy(e);
  for (auto& e : f->multi_ev)
    if (e) cudaEventDestroy(e);
  delete f;
}

int fsm_run(fsm_t f, const uint8_t* d_input, uint64_t len, const fsm_run_opts* opts, uint32_t* d_chunk_ends,
            fsm_result* out) {
  ApiScope api_scope_("fsm_run");
  if (!f || !out) return fail(FSM_EINVAL, "NULL handle/out");
  if (!d_input && len > 0) return fail(FSM_EINVAL, "NULL input");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  fsm_scheme scheme = o.scheme;
  if (scheme == FSM_SCHEME_AUTO) {
    if (!f->auto_selected) {
      fsm_run_opts so{};
      if (opts) so = *opts;
      so.scheme = FSM_SCHEME_SRE;
      fsm_scheme pick;
      rc = select_auto(f, d_input, len, &so);
      if (rc) return rc;
    }
    scheme = f->auto_scheme;
    if (scheme == FSM_SCHEME_ENUM && f->n + 1 > kEnumMax) scheme = FSM_SCHEME_SRE;
  }
  fsm_result r;
  uint32_t fin = 0;
  rc = run_core(f, d_input, len, o, scheme, f->img.q0t, d_chunk_ends, &r, &fin);
  if (rc) return rc;
  if (fin == f->n) return fail(FSM_ESYMBOL, "input symbol >= nsyms");
  r.final_state = f->inv[fin];
  r.accept = f->accept[r.final_state];
  *out = r;
  return FSM_OK;
}

int fsm_run_async(fsm_t f, const uint8_t* d_input, uint64_t len, const fsm_run_opts* opts, uint32_t* d_chunk_ends,
                  uint64_t* ticket) {
  ApiScope api_scope_("fsm_run_async");
  if (!f || !ticket) return fail(FSM_EINVAL, "NULL handle/ticket");
  if (!d_input && len > 0) return fail(FSM_EINVAL, "NULL input");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  fsm_scheme scheme = o.scheme;
  if (scheme == FSM_SCHEME_AUTO) {
    if (!f->auto_selected) {
      fsm_run_opts so{};
      if (opts) so = *opts;
      so.scheme = FSM_SCHEME_SRE;
      fsm_scheme pick;
      if ((rc = select_auto(f, d_input, len, &so))) return rc;
    }
    scheme = f->auto_scheme;
    if (scheme == FSM_SCHEME_ENUM && f->n + 1 > kEnumMax) scheme = FSM_SCHEME_SRE;
  }
  return run_enqueue(f, d_input, len, o, scheme, f->img.q0t, d_chunk_ends, ticket);
}

int fsm_wait(fsm_t f, uint64_t ticket, fsm_result* out) {
  ApiScope api_scope_("fsm_wait");
  if (!f || !out) return fail(FSM_EINVAL, "NULL handle/out");
  fsm_result r;
  uint32_t fin = 0;
  int rc = run_collect(f, ticket, &r, &fin);
  if (rc) return rc;
  if (fin == f->n) return fail(FSM_ESYMBOL, "input symbol >= nsyms");
  r.final_state = f->inv[fin];
  r.accept = f->accept[r.final_state];
  *out = r;
  return FSM_OK;
}

uint64_t fsm_batch_chunks(const uint64_t* h_offsets, uint32_t nstreams, uint32_t chunk_bytes) {
  if (!h_offsets) return 0;
  const uint32_t B = chunk_bytes ? chunk_bytes : 4096;
  uint64_t n = 0;
  for (uint32_t s = 0; s < nstreams; s++)
    if (h_offsets[s + 1] > h_offsets[s]) n += (h_offsets[s + 1] - h_offsets[s] + B - 1) / B;
  return n;
}

int fsm_run_batch(fsm_t f, const uint8_t* d_input, const uint64_t* h_offsets, uint32_t nstreams,
                  const fsm_run_opts* opts, uint32_t* d_final, uint64_t* d_count, uint32_t* d_chunk_ends,
                  fsm_batch_result* out) {
  ApiScope api_scope_("fsm_run_batch");
  if (!f || !out || !h_offsets) return fail(FSM_EINVAL, "NULL handle/offsets/out");
  std::memset(out, 0, sizeof(*out));
  if (nstreams == 0) return FSM_OK;
  if (!d_final || !d_count) return fail(FSM_EINVAL, "NULL d_final/d_count");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  if (o.L != 2) return fail(FSM_EUNSUPPORTED, "fsm_run_batch: lookback 2 only (the pair table, P:300)");
  const uint32_t B = o.B;
  std::vector<uint64_t> hb(2 * ((uint64_t)nstreams + 1));  // [offsets | chunk bases]
  uint64_t N = 0;
  for (uint32_t s = 0; s <= nstreams; s++) {
    if (s < nstreams && h_offsets[s + 1] < h_offsets[s]) return fail(FSM_EINVAL, "offsets must be non-decreasing");
    hb[s] = h_offsets[s];
    hb[nstreams + 1 + s] = N;
    if (s < nstreams) N += (h_offsets[s + 1] - h_offsets[s] + B - 1) / B;
  }
  if (N && !d_input) return fail(FSM_EINVAL, "NULL input");
  auto al = [](uint64_t b) { return (b + 255) & ~255ull; };
  const uint64_t need = al(hb.size() * 8) + 4 * al(N * 4 + 16) + al(gspec::batch_totals_bytes());
  if (f->batch_bytes < need) {
    CUDA_TRY(cudaStreamSynchronize(o.st));
    if (f->batch_base) cudaFree(f->batch_base);
    f->batch_base = nullptr;
    f->batch_bytes = 0;
    CUDA_TRY(cudaMalloc(&f->batch_base, need));
    f->batch_bytes = need;
  }
  if (!f->batch_ev[0]) {
    CUDA_TRY(cudaEventCreate(&f->batch_ev[0]));
    CUDA_TRY(cudaEventCreate(&f->batch_ev[1]));
  }
  uint8_t* p = reinterpret_cast<uint8_t*>(f->batch_base);
  uint64_t* d_off = reinterpret_cast<uint64_t*>(p);
  uint64_t* d_cb = d_off + nstreams + 1;
  p += al(hb.size() * 8);
  uint32_t* rs = reinterpret_cast<uint32_t*>(p); p += al(N * 4 + 16);
  uint32_t* re = reinterpret_cast<uint32_t*>(p); p += al(N * 4 + 16);
  uint32_t* rcn = reinterpret_cast<uint32_t*>(p); p += al(N * 4 + 16);
  uint32_t* cs = reinterpret_cast<uint32_t*>(p); p += al(N * 4 + 16);  // chunk -> stream
  void* tot = p;
  CUDA_TRY(cudaMemcpyAsync(d_off, hb.data(), hb.size() * 8, cudaMemcpyHostToDevice, o.st));
  CUDA_TRY(cudaMemsetAsync(tot, 0, gspec::batch_totals_bytes(), o.st));
  CUDA_TRY(cudaEventRecord(f->batch_ev[0], o.st));
  CUDA_TRY(gspec::launch_batch(f->img, d_input, d_off, d_cb, nstreams, N, B, cs, rs, re, rcn, d_final,
                               reinterpret_cast<unsigned long long*>(d_count), d_chunk_ends, tot, o.st, f->sm_count));
  CUDA_TRY(cudaEventRecord(f->batch_ev[1], o.st));
  uint64_t t[3] = {0, 0, 0};  // recoveries, reread, invalid (BatchTotals layout)
  CUDA_TRY(cudaMemcpyAsync(t, tot, sizeof(t), cudaMemcpyDeviceToHost, o.st));
  CUDA_TRY(cudaStreamSynchronize(o.st));
  out->nstreams = nstreams;
  out->nchunks = N;
  out->recoveries = t[0];
  out->reread_bytes = t[1];
  out->invalid_streams = t[2];
  cudaEventElapsedTime(&out->ms, f->batch_ev[0], f->batch_ev[1]);
  if (t[2]) return fail(FSM_ESYMBOL, "input symbol >= nsyms in some stream");
  return FSM_OK;
}

int fsm_run_multi(const fsm_t* fsms, uint32_t npairs, const uint8_t* const* d_inputs, const uint64_t* lens,
                  const fsm_run_opts* opts, uint32_t* h_final, uint64_t* h_count, fsm_multi_result* out) {
  ApiScope api_scope_("fsm_run_multi");
  if (out) std::memset(out, 0, sizeof(*out));
  if (npairs == 0) return FSM_OK;
  if (!fsms || !d_inputs || !lens || !h_final || !h_count) return fail(FSM_EINVAL, "NULL argument");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  if (o.L != 2) return fail(FSM_EUNSUPPORTED, "fsm_run_multi: lookback 2 only (the pair table, P:300)");
  std::vector<DevImage> imgs(npairs);
  std::vector<const uint8_t*> ins(npairs);
  std::vector<uint32_t> order;
  order.reserve(npairs);
  for (uint32_t i = 0; i < npairs; i++) {
    if (!fsms[i]) return fail(FSM_EINVAL, "NULL handle");
    if (!d_inputs[i] && lens[i]) return fail(FSM_EINVAL, "NULL input");
    imgs[i] = fsms[i]->img;
    ins[i] = d_inputs[i];
  }
  // group the pairs by table format: one launch per format present
  const int modes[5] = {MODE_U8, MODE_U16, MODE_U16H, MODE_U16D, MODE_U32};
  std::vector<std::pair<int, uint32_t>> groups;  // (mode, count)
  std::vector<uint32_t> smem_of;
  for (int m : modes) {
    uint32_t cnt = 0, sm = 0;
    for (uint32_t i = 0; i < npairs; i++)
      if ((int)imgs[i].mode == m) {
        order.push_back(i);
        cnt++;
        sm = std::max(sm, imgs[i].smem_table_bytes + ((m == MODE_U8 || m == MODE_U16D) ? 0u : 256u));  // walk.cuh smem_bytes_for
      }
    if (cnt) {
      groups.push_back({m, cnt});
      smem_of.push_back(sm);
    }
  }
  // device scratch: [images][inputs][lengths][pair order][finals][counts][stats]
  // scratch and events live in the first handle (device-bound, freed by fsm_free)
  void*& base = fsms[0]->multi_base;
  size_t& cap = fsms[0]->multi_cap;
  auto al = [](size_t b) { return (b + 255) & ~size_t(255); };
  const size_t b_img = al(sizeof(DevImage) * npairs), b_in = al(8 * npairs), b_len = al(8 * npairs),
               b_ord = al(4 * npairs), b_fin = al(4 * npairs), b_cnt = al(8 * npairs), b_st = 256;
  const size_t need = b_img + b_in + b_len + b_ord + b_fin + b_cnt + b_st;
  cudaStream_t st = o.st;
  if (cap < need) {
    CUDA_TRY(cudaStreamSynchronize(st));
    if (base) cudaFree(base);
    base = nullptr;
    cap = 0;
    CUDA_TRY(cudaMalloc(&base, need));
    cap = need;
  }
  uint8_t* p = static_cast<uint8_t*>(base);
  DevImage* d_imgs = reinterpret_cast<DevImage*>(p);
  const uint8_t** d_ins = reinterpret_cast<const uint8_t**>(p + b_img);
  uint64_t* d_lens = reinterpret_cast<uint64_t*>(p + b_img + b_in);
  uint32_t* d_ord = reinterpret_cast<uint32_t*>(p + b_img + b_in + b_len);
  uint32_t* d_fin = reinterpret_cast<uint32_t*>(p + b_img + b_in + b_len + b_ord);
  unsigned long long* d_cnt = reinterpret_cast<unsigned long long*>(p + b_img + b_in + b_len + b_ord + b_fin);
  unsigned long long* d_st = reinterpret_cast<unsigned long long*>(p + b_img + b_in + b_len + b_ord + b_fin + b_cnt);
  CUDA_TRY(cudaMemcpyAsync(d_imgs, imgs.data(), sizeof(DevImage) * npairs, cudaMemcpyHostToDevice, st));
  CUDA_TRY(cudaMemcpyAsync(d_ins, ins.data(), 8ull * npairs, cudaMemcpyHostToDevice, st));
  CUDA_TRY(cudaMemcpyAsync(d_lens, lens, 8ull * npairs, cudaMemcpyHostToDevice, st));
  CUDA_TRY(cudaMemcpyAsync(d_ord, order.data(), 4ull * npairs, cudaMemcpyHostToDevice, st));
  CUDA_TRY(cudaMemsetAsync(d_st, 0, 16, st));
  cudaEvent_t* ev = fsms[0]->multi_ev;
  for (int i = 0; i < 2; i++)
    if (!ev[i]) CUDA_TRY(cudaEventCreate(&ev[i]));
  CUDA_TRY(cudaEventRecord(ev[0], st));
  uint32_t off = 0;
  for (size_t g = 0; g < groups.size(); g++) {
    CUDA_TRY(launch_multi(groups[g].first, d_imgs, d_ins, d_lens, d_ord + off, groups[g].second, smem_of[g], o.B,
                          d_fin, d_cnt, d_st, st));
    off += groups[g].second;
  }
  CUDA_TRY(cudaEventRecord(ev[1], st));
  unsigned long long hst[2];
  CUDA_TRY(cudaMemcpyAsync(h_final, d_fin, 4ull * npairs, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaMemcpyAsync(h_count, d_cnt, 8ull * npairs, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaMemcpyAsync(hst, d_st, 16, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaStreamSynchronize(st));
  if (out) {
    out->rewalks = hst[0];
    out->rounds = hst[1];
    cudaEventElapsedTime(&out->ms, ev[0], ev[1]);
  }
  for (uint32_t i = 0; i < npairs; i++)
    if (h_final[i] == 0xFFFFFFFFu) return fail(FSM_ESYMBOL, "input symbol >= nsyms in some stream");
  return FSM_OK;
}

int fsm_run_literal(fsm_t f, const uint8_t* d_input, uint64_t len, const fsm_run_opts* opts,
                    uint32_t* d_chunk_ends, fsm_result* out) {
  ApiScope api_scope_("fsm_run_literal");
  if (!f || !out) return fail(FSM_EINVAL, "NULL handle/out");
  if (!d_input && len > 0) return fail(FSM_EINVAL, "NULL input");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  if (o.L != 2) return fail(FSM_EUNSUPPORTED, "fsm_run_literal: lookback 2 only (the pair table, P:300)");
  const uint64_t N = fsm_num_chunks(len, o.B);
  if (N > literal_max_chunks()) return fail(FSM_EUNSUPPORTED, "paper-literal kernel: at most 1024 chunks (one CTA)");
  // SRE (Alg. 3, the default for AUTO), RR (Alg. 4) or NF (Alg. 5)
  const fsm_scheme lscheme = (o.scheme == FSM_SCHEME_RR || o.scheme == FSM_SCHEME_NF) ? o.scheme : FSM_SCHEME_SRE;
  if (o.scheme != FSM_SCHEME_AUTO && o.scheme != lscheme)
    return fail(FSM_EUNSUPPORTED, "paper-literal kernel: SRE, RR or NF (Alg. 3-5)");
  std::memset(out, 0, sizeof(*out));
  out->nchunks = N;
  out->scheme_used = lscheme;
  uint32_t fin = f->img.q0t;
  if (N) {
    if ((rc = ensure_ctl(f))) return rc;
    CUDA_TRY(cudaStreamSynchronize(o.st));  // queued runs may still use the record store
    if ((rc = ensure_records(f, N))) return rc;
    RunParams rp{};
    rp.in = d_input;
    rp.q0t = f->img.q0t;
    rp.len = len;
    rp.B = o.B;
    rp.N = N;
    rp.scheme = lscheme;
    rp.k = 1;
    rp.qs_cap = o.qs_cap;
    rp.vr_end = o.vr_end;
    rp.vr_oth = o.vr_oth;
    for (auto& e : f->batch_ev)
      if (!e) CUDA_TRY(cudaEventCreate(&e));
    cudaEvent_t e0 = f->batch_ev[0], e1 = f->batch_ev[1];
    CUDA_TRY(cudaMemsetAsync(f->d_ctl, 0, sizeof(Ctl), o.st));
    CUDA_TRY(cudaEventRecord(e0, o.st));
    CUDA_TRY(launch_literal_sre(f->img, rp, f->rs, f->d_ctl, d_chunk_ends, o.st));
    CUDA_TRY(cudaEventRecord(e1, o.st));
    Ctl h;
    CUDA_TRY(cudaMemcpyAsync(&h, f->d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, o.st));
    CUDA_TRY(cudaStreamSynchronize(o.st));
    fill_result_stats(out, h);
    out->accept_count = h.accept_count;
    float t = 0;
    cudaEventElapsedTime(&t, e0, e1);
    out->ms_verify = t;
    out->kernel_launches = 1;
    fin = h.xfin;
  }
  if (fin == f->n) return fail(FSM_ESYMBOL, "input symbol >= nsyms");
  out->final_state = f->inv[fin];
  out->accept = f->accept[out->final_state];
  return FSM_OK;
}

int fsm_run_host(fsm_t f, const uint8_t* h_input, uint64_t len, const fsm_run_opts* opts, uint32_t* h_chunk_ends,
                 fsm_result* out) {
  ApiScope api_scope_("fsm_run_host");
  if (!f || !out) return fail(FSM_EINVAL, "NULL handle/out");
  if (!h_input && len > 0) return fail(FSM_EINVAL, "NULL input");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  const uint64_t N = fsm_num_chunks(len, o.B);
  if (f->h_in_cap < len) {
    if (f->h_dev_in) cudaFree(f->h_dev_in);
    f->h_dev_in = nullptr;
    f->h_in_cap = 0;
    CUDA_TRY(cudaMalloc(&f->h_dev_in, len + 16));
    f->h_in_cap = len;
  }
  if (h_chunk_ends && f->h_ce_cap < N) {
    if (f->h_dev_ce) cudaFree(f->h_dev_ce);
    f->h_dev_ce = nullptr;
    f->h_ce_cap = 0;
    CUDA_TRY(cudaMalloc(&f->h_dev_ce, N * 4 + 16));
    f->h_ce_cap = N;
  }
  if (len) CUDA_TRY(cudaMemcpyAsync(f->h_dev_in, h_input, len, cudaMemcpyHostToDevice, o.st));
  rc = fsm_run(f, (const uint8_t*)f->h_dev_in, len, opts, h_chunk_ends ? (uint32_t*)f->h_dev_ce : nullptr, out);
  if (rc) return rc;
  if (h_chunk_ends && N) {
    CUDA_TRY(cudaMemcpyAsync(h_chunk_ends, f->h_dev_ce, N * 4, cudaMemcpyDeviceToHost, o.st));
    CUDA_TRY(cudaStreamSynchronize(o.st));
  }
  return FSM_OK;
}

int fsm_select_scheme(fsm_t f, const uint8_t* d_sample, uint64_t len, const fsm_run_opts* opts, fsm_scheme* outp,
                      fsm_features* feat) {
  ApiScope api_scope_("fsm_select_scheme");
  if (!f || !outp) return fail(FSM_EINVAL, "NULL handle/out");
  if (!d_sample && len > 0) return fail(FSM_EINVAL, "NULL sample");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  // Reading R20 ("a randomly selected 1 MB trace"; "similarity of speculation
  // results over different portions"): a trace longer than 1 MiB is profiled on 8
  // portions of 128 KiB spread evenly from its start to its end (portion i at
  // i (len - 128 KiB) / 7, 4 KiB-aligned), gathered into one 1 MiB sample, so the
  // input-sensitivity feature compares different portions of the stream.
  constexpr uint64_t kSlice = 128 << 10, kSample = 8 * kSlice;
  const uint64_t stream_len = len;  // the chunk-size rule's occupancy bound (R29)
  if (len > kSample) {
    if (!f->prof_buf) CUDA_TRY(cudaMalloc(&f->prof_buf, kSample));
    for (uint64_t i = 0; i < 8; i++) {
      const uint64_t off = (i * (len - kSlice) / 7) & ~4095ull;
      CUDA_TRY(cudaMemcpyAsync(f->prof_buf + i * kSlice, d_sample + off, kSlice, cudaMemcpyDeviceToDevice, o.st));
    }
    d_sample = f->prof_buf;
    len = kSample;
  }
  // 1. true chunk starts by an exact scheme on the sample
  fsm_result r;
  uint32_t fin = 0;
  rc = run_core(f, d_sample, len, o, FSM_SCHEME_SRE, f->img.q0t, nullptr, &r, &fin);
  if (rc) return rc;
  const uint64_t N = r.nchunks;
  // 2. features on the device
  const uint32_t words = (f->n + 1 + 31) / 32;
  // convergence windows (R29): p = 4096 j, j mod 32 in [1, 28], p + kConvMax <= len
  constexpr uint32_t kConvMax = 16384;
  uint32_t nwin = 0;
  for (uint64_t j = 1; j * 4096 + kConvMax <= len; j++) nwin += (j % 32 >= 1 && j % 32 <= 28);
  const size_t conv_off = 32 * 8 + 64ull * words * 4 + 64;
  const size_t need = conv_off + 4ull * nwin + 16;
  if (f->feat_bytes < need) {
    if (f->feat_base) cudaFree(f->feat_base);
    f->feat_base = nullptr;
    f->feat_bytes = 0;
    CUDA_TRY(cudaMalloc(&f->feat_base, need));
    f->feat_bytes = need;
  }
  unsigned long long* d_counts = (unsigned long long*)f->feat_base;  // [0..18) + uniq at [20]
  uint32_t* d_seen = (uint32_t*)((uint8_t*)f->feat_base + 32 * 8);
  CUDA_TRY(cudaMemsetAsync(f->feat_base, 0, need, o.st));
  fsm_features ft{};
  ft.nstates = f->n;
  if (len > 0) {
    CUDA_TRY(launch_features_raw(f->img, f->d_ttc, d_sample, len, o.B, N, f->rs.x, o.k, o.qs_cap, d_counts, d_seen,
                                 d_counts + 20, o.st));
    unsigned long long h[32];
    CUDA_TRY(cudaMemcpyAsync(h, d_counts, sizeof(h), cudaMemcpyDeviceToHost, o.st));
    CUDA_TRY(cudaStreamSynchronize(o.st));
    if (N > 1) {
      ft.acc1 = (double)h[16] / (double)(N - 1);
      ft.acck = (double)h[17] / (double)(N - 1);
      double mx = -1, mn = 2;
      for (int s = 0; s < 8; s++) {
        if (!h[8 + s]) continue;
        const double a = (double)h[s] / (double)h[8 + s];
        mx = std::max(mx, a);
        mn = std::min(mn, a);
      }
      ft.input_sensitivity = mx >= 0 ? mx - mn : 0;
    }
    if (len >= 10) ft.uniq10 = (double)h[20] / 64.0;
  }
  // R29: convergence lengths of the lookback image -> recommended chunk size
  ft.chunk_bytes = 4096;
  if (nwin > 0) {
    uint32_t* d_conv = reinterpret_cast<uint32_t*>(static_cast<uint8_t*>(f->feat_base) + conv_off);
    CUDA_TRY(launch_feat_conv(f->img, f->d_ttc, d_sample, nwin, kConvMax, d_conv, o.st));
    std::vector<uint32_t> dv(nwin);
    CUDA_TRY(cudaMemcpyAsync(dv.data(), d_conv, 4ull * nwin, cudaMemcpyDeviceToHost, o.st));
    CUDA_TRY(cudaStreamSynchronize(o.st));
    double* conv[3] = {&ft.conv4k, &ft.conv8k, &ft.conv16k};
    for (uint32_t W = 4096, i = 0; W <= kConvMax; W *= 2, i++) {
      uint64_t k = 0;
      for (uint32_t d : dv) k += d <= W;
      *conv[i] = (double)k / nwin;  // exact at 3/4 (0.75 is representable)
    }
    ft.chunk_bytes = fsm_chunk_for(&ft, stream_len);
  }
  const fsm_scheme pick = tree_select(ft, f->n);
  if (N > 1) f->acc1_hint = ft.acc1;
  if (nwin > 0) f->conv_hint = ft.conv16k;  // R30: no window converged within 16 KiB -> no checkpoints
  f->auto_scheme = pick;
  f->auto_selected = true;
  *outp = pick;
  if (feat) *feat = ft;
  return FSM_OK;
}

uint32_t fsm_chunk_for(const fsm_features* ft, uint64_t stream_len) {
  if (!ft) return 4096;
  const uint64_t min_chunks = (uint64_t)device_sms() * 768;  // 24 warps per SM of one-chunk lanes
  const double conv[3] = {ft->conv4k, ft->conv8k, ft->conv16k};
  for (uint32_t W = 4096, i = 0; i < 3; W *= 2, i++)
    if (conv[i] >= 0.75 && (W == 4096 || stream_len / W >= min_chunks)) return W;
  return 4096;
}

int fsm_get_transform(fsm_t f, uint32_t* perm, uint32_t* inv, uint64_t* freq, uint32_t* mode, uint32_t* hot_rows,
                      uint32_t* nclasses) {
  if (!f) return fail(FSM_EINVAL, "NULL handle");
  if (perm) std::copy(f->perm.begin(), f->perm.end(), perm);
  if (inv) std::copy(f->inv.begin(), f->inv.end(), inv);
  if (freq) std::copy(f->freq.begin(), f->freq.end(), freq);
  if (mode) *mode = f->img.mode == MODE_U16H ? (uint32_t)MODE_U16 : f->img.mode == MODE_U16D ? 4u : f->img.mode;
  if (hot_rows) *hot_rows = f->img.mode == MODE_U16D ? f->img.HC1 / f->img.C - 1 : f->img.H;  // full real rows
  if (nclasses) *nclasses = f->img.C;
  return FSM_OK;
}

int fsm_get_qs(fsm_t f, uint8_t a, uint8_t b, uint32_t* qs, uint32_t* qs_len, uint32_t* image_size) {
  if (!f) return fail(FSM_EINVAL, "NULL handle");
  const uint64_t pair = (uint64_t)f->cls[a] * f->img.C + f->cls[b];
  uint8_t l = 0;
  uint32_t im = 0;
  CUDA_TRY(cudaMemcpy(&l, f->img.qs2_len + pair, 1, cudaMemcpyDeviceToHost));
  CUDA_TRY(cudaMemcpy(&im, f->img.qs2_img + pair, 4, cudaMemcpyDeviceToHost));
  if (qs) CUDA_TRY(cudaMemcpy(qs, f->img.qs2 + pair * kQsMax, 4 * l, cudaMemcpyDeviceToHost));
  if (qs_len) *qs_len = l;
  if (image_size) *image_size = im;
  return FSM_OK;
}

int fsm_get_records(fsm_t f, uint64_t N, uint32_t* start, uint32_t* end, uint32_t* cnt, uint32_t* n_end,
                    uint32_t* n_oth, uint32_t* x) {
  if (!f || !f->rs_base || N > f->rs_cap) return fail(FSM_EINVAL, "no records for that many chunks");
  const RecStore& r = f->rs;
  for (uint32_t s = 0; s < kSlots; s++) {
    if (start) CUDA_TRY(cudaMemcpy(start + s * N, r.start + s * r.cap, 4 * N, cudaMemcpyDeviceToHost));
    if (end) CUDA_TRY(cudaMemcpy(end + s * N, r.end + s * r.cap, 4 * N, cudaMemcpyDeviceToHost));
    if (cnt) CUDA_TRY(cudaMemcpy(cnt + s * N, r.cnt + s * r.cap, 4 * N, cudaMemcpyDeviceToHost));
  }
  if (n_end) CUDA_TRY(cudaMemcpy(n_end, r.n_end, 4 * N, cudaMemcpyDeviceToHost));
  if (n_oth) CUDA_TRY(cudaMemcpy(n_oth, r.n_oth, 4 * N, cudaMemcpyDeviceToHost));
  if (x) CUDA_TRY(cudaMemcpy(x, r.x, 4 * (N + 1), cudaMemcpyDeviceToHost));
  return FSM_OK;
}

int fsm_get_phase_times(fsm_t f, double* us, uint32_t* n) {
  if (!f || !n) return fail(FSM_EINVAL, "NULL handle/n");
  const uint32_t k = f->last_nstamp;
  if (us)
    for (uint32_t i = 0; i < k; i++) us[i] = (f->last_stamp[i] - f->last_stamp[0]) * 1e-3;
  *n = k;
  return FSM_OK;
}

int fsm_get_timeline(fsm_t f, double* us) {
  if (!f || !us) return fail(FSM_EINVAL, "NULL handle/us");
  const uint64_t* t = f->last_tl;
  const bool ok = t[0] && t[1] >= t[0] && t[2] >= t[1] && t[3] >= t[2];
  for (int i = 0; i < 3; i++) us[i] = ok ? (t[i + 1] - t[i]) * 1e-3 : -1.0;
  return FSM_OK;
}

uint64_t fsm_map_bytes(fsm_t f) {
  if (!f) return 0;
  const uint64_t nt = f->n + 1;
  return ((nt * 4 + 7) & ~7ull) + nt * 8;
}

}  // extern "C"

// ---- multi-GPU shard steps: implemented in shard.cpp ----

namespace {

constexpr uint32_t kFuseChunks = 8;   // path-fusion window (chunks) before falling back
constexpr uint32_t kNoState = 0xFFFFFFFFu;

uint64_t map_cnt_off(uint32_t nt) { return ((uint64_t)nt * 4 + 7) & ~7ull; }
uint64_t map_bytes_nt(uint32_t nt) { return map_cnt_off(nt) + (uint64_t)nt * 8; }

struct ShardScratch {
  uint32_t *mark, *cand, *info, *states, *grp, *pfinal;
  unsigned long long *prefix, *pcount;
};

int ensure_shard(fsm_t f, ShardScratch* s) {
  const uint64_t nt = f->n + 1;
  const uint64_t words = nt * 2 + 16 + kFuseChunks * nt + nt * 2 + nt * 2 + nt * 2 + 64;
  const size_t need = words * 8;
  if (f->shard_bytes < need) {
    if (f->shard_base) cudaFree(f->shard_base);
    f->shard_base = nullptr;
    f->shard_bytes = 0;
    CUDA_TRY(cudaMalloc(&f->shard_base, need));
    f->shard_bytes = need;
  }
  uint64_t* p = reinterpret_cast<uint64_t*>(f->shard_base);
  s->prefix = reinterpret_cast<unsigned long long*>(p); p += nt;
  s->pcount = reinterpret_cast<unsigned long long*>(p); p += nt;
  uint32_t* u = reinterpret_cast<uint32_t*>(p);
  s->mark = u; u += nt;
  s->cand = u; u += nt;
  s->info = u; u += 32;
  s->grp = u; u += nt;
  s->pfinal = u; u += nt;
  s->states = u;
  return FSM_OK;
}

int resolve_scheme(fsm_t f, const uint8_t* d_in, uint64_t len, const fsm_run_opts* opts, const Opts& o,
                   fsm_scheme* out) {
  fsm_scheme scheme = o.scheme;
  if (scheme == FSM_SCHEME_AUTO) {
    if (!f->auto_selected) {
      fsm_run_opts so{};
      if (opts) so = *opts;
      so.scheme = FSM_SCHEME_SRE;
      fsm_scheme pick;
      int rc = select_auto(f, d_in, len, &so);
      if (rc) return rc;
    }
    scheme = f->auto_scheme;
  }
  if (scheme == FSM_SCHEME_ENUM && f->n + 1 > kEnumMax) scheme = FSM_SCHEME_SRE;
  *out = scheme;
  return FSM_OK;
}


int ensure_enum_scratch(fsm_t f, uint64_t nsub) {
  const uint64_t need = enum_scratch_bytes(nsub);
  if (f->enum_bytes < need) {
    if (f->enum_base) cudaFree(f->enum_base);
    f->enum_base = nullptr;
    f->enum_bytes = 0;
    CUDA_TRY(cudaMalloc(&f->enum_base, need));
    f->enum_bytes = need;
  }
  if (!f->d_small) CUDA_TRY(cudaMalloc(&f->d_small, 64 * sizeof(uint32_t)));
  return FSM_OK;
}

}  // namespace

extern "C" {

int shard_map_impl(fsm_t f, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback, uint32_t lb_len,
                   const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local, bool exact);

int fsm_shard_map(fsm_t f, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback, uint32_t lb_len,
                  const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local) {
  ApiScope api_scope_("fsm_shard_map");
  return shard_map_impl(f, d_shard, len, d_lookback, lb_len, opts, d_map, d_chunk_ends_local,
                        f && f->shard_prefer_exact);
}

int fsm_shard_map_exact(fsm_t f, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback, uint32_t lb_len,
                        const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local) {
  ApiScope api_scope_("fsm_shard_map_exact");
  return shard_map_impl(f, d_shard, len, d_lookback, lb_len, opts, d_map, d_chunk_ends_local, true);
}

int shard_map_body(fsm_t f, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback, uint32_t lb_len,
                   const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local, bool exact);

// A failed map must not strand the other ranks in the exchange (they are already
// waiting in the allgather): the failing rank publishes an error map, still takes part
// in the collective, and every rank's fsm_shard_finish returns this rank's status.
int shard_map_impl(fsm_t f, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback, uint32_t lb_len,
                   const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local, bool exact) {
  const int rc = shard_map_body(f, d_shard, len, d_lookback, lb_len, opts, d_map, d_chunk_ends_local, exact);
  if (rc != FSM_OK && f && d_map) {
    cudaStream_t st = opts ? reinterpret_cast<cudaStream_t>(opts->stream) : nullptr;
    const uint32_t nt = f->n + 1;
    uint32_t* mend = reinterpret_cast<uint32_t*>(d_map);
    unsigned long long* mcnt =
        reinterpret_cast<unsigned long long*>(reinterpret_cast<uint8_t*>(d_map) + map_cnt_off(nt));
    if (launch_map_error(mend, mcnt, nt, (uint32_t)(-rc), st) == cudaSuccess) f->shard_mode = 4;
  }
  return rc;
}

int shard_map_body(fsm_t f, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback, uint32_t lb_len,
                   const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local, bool exact) {
  if (!f || !d_map) return fail(FSM_EINVAL, "NULL handle/map");
  if (!d_shard && len > 0) return fail(FSM_EINVAL, "NULL shard");
  if (lb_len > 16 || (lb_len && !d_lookback)) return fail(FSM_EINVAL, "lookback_len must be <= 16 with bytes");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  fsm_scheme scheme;
  if ((rc = resolve_scheme(f, d_shard, len, opts, o, &scheme))) return rc;
  ShardScratch S;
  if ((rc = ensure_shard(f, &S))) return rc;
  if ((rc = ensure_ctl(f))) return rc;
  if (!f->d_small) CUDA_TRY(cudaMalloc(&f->d_small, 64 * sizeof(uint32_t)));
  const uint32_t nt = f->n + 1;
  const uint64_t N = (len + o.B - 1) / o.B;
  uint32_t* mend = reinterpret_cast<uint32_t*>(d_map);
  unsigned long long* mcnt = reinterpret_cast<unsigned long long*>(reinterpret_cast<uint8_t*>(d_map) + map_cnt_off(nt));
  CUDA_TRY(launch_map_init(mend, mcnt, nt, o.st));
  // 1. candidate start states: the lookback image or q0 for the first shard
  f->shard_in = d_shard;
  f->shard_len = len;
  f->shard_nj = 0;
  f->shard_scheme = scheme;
  f->shard_dist.clear();
  uint32_t* d_ncand = S.info + 8;
  uint32_t* d_unmerged = S.info + 9;
  long long* dcnt = reinterpret_cast<long long*>(S.prefix);
  if (lb_len == 0) {
    CUDA_TRY(launch_set_u32(S.cand, f->img.q0t, d_ncand, 1, o.st));
    CUDA_TRY(cudaMemsetAsync(S.grp, 0, 4, o.st));
    CUDA_TRY(cudaMemsetAsync(dcnt, 0, 8, o.st));
  } else {
    CUDA_TRY(launch_shard_image(f->img, f->d_ttc, d_lookback, lb_len, S.mark, S.cand, d_ncand, o.st));
  }
  // 2a. fast path: fuse every candidate with the path of cand[0] (P:427 path
  // fusion); the shard then runs once, from cand[0], through the normal pipeline.
  // Speculative (default): no host check — the pipeline is queued at once and the map
  // kernel marks the map invalid if some candidate did not merge; the composition then
  // reports FSM_EAGAIN on every rank and all ranks redo fsm_shard_map_exact (DESIGN.md
  // §8).  Exact: one host check (did every candidate merge?), else the fallbacks below.
  if (N > 0 && len > 0) {
    uint32_t h2[2] = {1, 0};
    if (lb_len != 0) {
      CUDA_TRY(cudaMemsetAsync(d_unmerged, 0, 4, o.st));
      CUDA_TRY(launch_shard_fuse_ref(f->img, d_shard, len, o.B, S.cand, d_ncand, kFuseChunks, S.states, S.grp, dcnt,
                                     d_unmerged, o.st));
      if (exact) {
        CUDA_TRY(cudaMemcpyAsync(h2, d_ncand, 8, cudaMemcpyDeviceToHost, o.st));
        CUDA_TRY(cudaStreamSynchronize(o.st));
      }
    }
    f->shard_ncand = h2[0];  // (speculative: not read on the host in fused mode)
    if (h2[1] == 0) {
      if (f->shard_ticket) {  // a previous shard run that was never finished
        fsm_result rr;
        uint32_t ff;
        run_collect(f, f->shard_ticket, &rr, &ff);
        f->shard_ticket = 0;
      }
      if ((rc = run_enqueue(f, d_shard, len, o, scheme, f->img.q0t, d_chunk_ends_local, &f->shard_ticket, S.cand)))
        return rc;
      if (f->p2p_pub) {  // peer-memory exchange: the map kernel also sends the map (p2p.cu)
        const auto& pp = *f->p2p_pub;
        CUDA_TRY(launch_map_fused_publish(S.cand, d_ncand, dcnt, &f->d_ctl->xfin,
                                          reinterpret_cast<const unsigned long long*>(&f->d_ctl->accept_count), mend,
                                          mcnt, (lb_len != 0 && !exact) ? d_unmerged : nullptr, pp.mapb, pp.peers,
                                          pp.G, pp.rank, pp.set, pp.seq, o.st));
        f->p2p_published = true;
      } else {
        CUDA_TRY(launch_map_fused(S.cand, d_ncand, dcnt, &f->d_ctl->xfin,
                                  reinterpret_cast<const unsigned long long*>(&f->d_ctl->accept_count), mend, mcnt,
                                  (lb_len != 0 && !exact) ? d_unmerged : nullptr, o.st));
      }
      f->shard_mode = 3;
      return FSM_OK;
    }
  }
  // fallback: host-driven fusion / enumeration (candidate list needed on the host)
  uint32_t ncand = 1;
  CUDA_TRY(cudaMemcpyAsync(&ncand, d_ncand, 4, cudaMemcpyDeviceToHost, o.st));
  CUDA_TRY(cudaStreamSynchronize(o.st));
  f->shard_cand.resize(ncand);
  CUDA_TRY(cudaMemcpy(f->shard_cand.data(), S.cand, 4ull * ncand, cudaMemcpyDeviceToHost));
  f->shard_ncand = ncand;
  f->shard_grp.assign(ncand, 0);
  std::vector<uint32_t> last(f->shard_cand);
  uint32_t nj = 0;
  bool merged = ncand == 1;
  // 2. path fusion over the first chunks
  if (!merged && N > 0 && ncand <= 1024) {
    const uint32_t W = (uint32_t)std::min<uint64_t>(kFuseChunks, N);
    CUDA_TRY(launch_shard_fuse(f->img, d_shard, len, o.B, S.cand, ncand, W, S.states, S.prefix, S.info, o.st));
    uint32_t info[2];
    CUDA_TRY(cudaMemcpyAsync(info, S.info, 8, cudaMemcpyDeviceToHost, o.st));
    CUDA_TRY(cudaStreamSynchronize(o.st));
    nj = info[1];
    merged = info[0] != kNoState;
    CUDA_TRY(cudaMemcpy(last.data(), S.states + (uint64_t)(nj - 1) * ncand, 4ull * ncand, cudaMemcpyDeviceToHost));
  }
  f->shard_nj = nj;
  const uint64_t off = (uint64_t)nj * o.B, rest = len - std::min<uint64_t>(len, off);
  if (merged || (nt > kEnumMax)) {
    // distinct surviving paths; each runs the speculative pipeline over the rest
    std::vector<uint32_t>& D = f->shard_dist;
    for (uint32_t i = 0; i < ncand; i++) {
      auto it = std::find(D.begin(), D.end(), last[i]);
      if (it == D.end()) {
        D.push_back(last[i]);
        f->shard_grp[i] = (uint32_t)D.size() - 1;
      } else {
        f->shard_grp[i] = (uint32_t)(it - D.begin());
      }
    }
    // more than kMaxMulti non-merging paths (a non-convergent DFA too large for ENUM):
    // still exact, at the cost of one pipeline per surviving path
    std::vector<uint32_t> fin(D.size());
    std::vector<unsigned long long> cnt(D.size());
    for (size_t d = 0; d < D.size(); d++) {
      fsm_result r;
      uint32_t ft = D[d];
      if (rest) {
        const bool write_ce = D.size() == 1 && d_chunk_ends_local;
        rc = run_core(f, d_shard + off, rest, o, scheme, D[d], write_ce ? d_chunk_ends_local + nj : nullptr, &r, &ft);
        if (rc) return rc;
        cnt[d] = r.accept_count;
      } else {
        cnt[d] = 0;
      }
      fin[d] = ft;
    }
    f->shard_mode = D.size() == 1 ? 0 : 2;
    CUDA_TRY(cudaMemcpyAsync(S.grp, f->shard_grp.data(), 4ull * ncand, cudaMemcpyHostToDevice, o.st));
    CUDA_TRY(cudaMemcpyAsync(S.pfinal, fin.data(), 4ull * fin.size(), cudaMemcpyHostToDevice, o.st));
    CUDA_TRY(cudaMemcpyAsync(S.pcount, cnt.data(), 8ull * cnt.size(), cudaMemcpyHostToDevice, o.st));
    CUDA_TRY(launch_map_write(S.cand, ncand, S.grp, nj ? S.prefix : nullptr, S.pfinal, S.pcount, mend, mcnt, o.st));
    CUDA_TRY(cudaStreamSynchronize(o.st));
    if (nj && d_chunk_ends_local && f->shard_mode == 0)
      CUDA_TRY(launch_fix_prefix(S.states, ncand, 0, nj, f->img.inv, d_chunk_ends_local, o.st));
  } else {
    // non-convergent small DFA: enumerate the whole shard
    f->shard_mode = 1;
    f->shard_E = enum_sub_bytes(o.B, len);
    const uint64_t nsub = (len + f->shard_E - 1) / f->shard_E;
    if ((rc = ensure_enum_scratch(f, nsub))) return rc;
    RunParams rp{};
    rp.in = d_shard;
    rp.q0t = f->img.q0t;
    rp.len = len;
    rp.B = o.B;
    rp.N = N;
    const uint8_t* topM = nullptr;
    const uint64_t* topC = nullptr;
    CUDA_TRY(launch_enum_full(f->img, rp, f->shard_E, f->enum_base, nullptr, f->d_ctl, f->d_small, o.st, f->sm_count,
                              1, &topM, &topC));
    CUDA_TRY(launch_map_enum(topM, reinterpret_cast<const unsigned long long*>(topC), nt, mend, mcnt, o.st));
  }
  CUDA_TRY(cudaStreamSynchronize(o.st));
  return FSM_OK;
}

int fsm_shard_finish(fsm_t f, const void* d_maps, uint32_t G, uint32_t rank, const fsm_run_opts* opts,
                     uint32_t* d_chunk_ends_local, fsm_result* out) {
  ApiScope api_scope_("fsm_shard_finish");
  if (!f || !d_maps || !out || rank >= G) return fail(FSM_EINVAL, "bad finish arguments");
  if (f->shard_mode < 0) return fail(FSM_EINVAL, "fsm_shard_map was not called");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  const uint32_t nt = f->n + 1;
  if (!f->d_small) CUDA_TRY(cudaMalloc(&f->d_small, 64 * sizeof(uint32_t)));  // (a map that failed early)
  CUDA_TRY(launch_compose(reinterpret_cast<const uint8_t*>(d_maps), G, map_bytes_nt(nt), map_cnt_off(nt), f->img.q0t,
                          rank, f->d_small, o.st, f->p2p_wait ? f->p2p_wait->flags : nullptr,
                          f->p2p_wait ? f->p2p_wait->seq : 0, f->p2p_wait ? f->p2p_wait->status : nullptr));
  if (f->shard_mode == 3) {
    // fused mode: this rank's chunk ends before the merge point are fixed on the device
    ShardScratch S3;
    if ((rc = ensure_shard(f, &S3))) return rc;
    CUDA_TRY(cudaMemsetAsync(f->d_small + 5, 0, 4, o.st));
    if (d_chunk_ends_local && f->shard_len)
      CUDA_TRY(launch_fix_prefix_fused(S3.states, S3.cand, S3.info + 8, S3.grp, f->d_small, f->img.inv, f->n,
                                       d_chunk_ends_local, f->d_small + 5, o.st));
  }
  uint32_t h[6] = {0, 0, 0, 0, 0, 0};
  CUDA_TRY(cudaMemcpyAsync(h, f->d_small, sizeof(h), cudaMemcpyDeviceToHost, o.st));
  CUDA_TRY(cudaStreamSynchronize(o.st));
  if (f->shard_mode == 3 && f->shard_ticket) {
    fsm_result rr;
    uint32_t ff;
    rc = run_collect(f, f->shard_ticket, &rr, &ff);  // already complete: frees the ring slot
    f->shard_ticket = 0;
    if (rc) return rc;
  }
  if (h[2] == 3) {  // some rank's map failed: every rank returns that rank's status
    const int code = -(int)h[3];
    char msg[96];
    std::snprintf(msg, sizeof(msg), "fsm_shard_map failed on rank %u (%s)", h[4], fsm_strerror(code));
    return fail(code < 0 ? code : FSM_EINVAL, msg);
  }
  if (h[2] == 2) {
    f->shard_prefer_exact = true;  // this DFA's shards do not merge early: skip speculation from now on
    return fail(FSM_EAGAIN, "a rank's speculative shard map was invalid: every rank redoes fsm_shard_map_exact");
  }
  if (f->shard_mode == 4) return fail(FSM_EINVAL, "this rank's fsm_shard_map failed");
  if (h[2] || (f->shard_mode == 3 && h[5])) return fail(FSM_EINVAL, "a shard start state is outside its candidate set");
  const uint32_t srank = h[0], fin = h[1];
  const uint64_t count = (uint64_t)h[3] | ((uint64_t)h[4] << 32);
  const uint64_t N = (f->shard_len + o.B - 1) / o.B;
  ShardScratch S;
  if ((rc = ensure_shard(f, &S))) return rc;
  if (d_chunk_ends_local && N && srank != f->n) {  // poison start: FSM_ESYMBOL below
    if (f->shard_mode == 1) {
      RunParams rp{};
      rp.in = f->shard_in;
      rp.q0t = srank;
      rp.len = f->shard_len;
      rp.B = o.B;
      rp.N = N;
      CUDA_TRY(launch_enum_full(f->img, rp, f->shard_E, f->enum_base, d_chunk_ends_local, f->d_ctl, f->d_small + 8,
                                o.st, f->sm_count, 2));
    } else if (f->shard_mode == 3) {
      (void)srank;  // located on the device
    } else {
      auto it = std::find(f->shard_cand.begin(), f->shard_cand.end(), srank);
      if (it == f->shard_cand.end()) return fail(FSM_EINVAL, "rank start not among its candidates");
      const uint32_t ci = (uint32_t)(it - f->shard_cand.begin());
      if (f->shard_nj) CUDA_TRY(launch_fix_prefix(S.states, f->shard_ncand, ci, f->shard_nj, f->img.inv,
                                                  d_chunk_ends_local, o.st));
      if (f->shard_mode == 2) {
        const uint64_t off = (uint64_t)f->shard_nj * o.B;
        if (off < f->shard_len) {
          fsm_result r;
          uint32_t ft;
          rc = run_core(f, f->shard_in + off, f->shard_len - off, o, f->shard_scheme, f->shard_dist[f->shard_grp[ci]],
                        d_chunk_ends_local + f->shard_nj, &r, &ft);
          if (rc) return rc;
        }
      }
    }
    CUDA_TRY(cudaStreamSynchronize(o.st));
  }
  std::memset(out, 0, sizeof(*out));
  out->nchunks = N;
  out->scheme_used = f->shard_scheme;
  if (fin == f->n) return fail(FSM_ESYMBOL, "input symbol >= nsyms");
  out->final_state = f->inv[fin];
  out->accept = f->accept[out->final_state];
  out->accept_count = count;
  return FSM_OK;
}

// Asynchronous finish (stream-ordered): in the fused mode the composition, the prefix
// fix-up and a copy of the 6 result words into a pinned ring slot are queued and the call
// returns a ticket at once; the modes whose fix-up runs on the host finish synchronously
// (the ticket then carries the outcome).  fsm_shard_wait blocks for a ticket and decodes.
int fsm_shard_finish_async(fsm_t f, const void* d_maps, uint32_t G, uint32_t rank, const fsm_run_opts* opts,
                           uint32_t* d_chunk_ends_local, uint64_t* ticket) {
  ApiScope api_scope_("fsm_shard_finish_async");
  if (!f || !d_maps || !ticket || rank >= G) return fail(FSM_EINVAL, "bad finish arguments");
  if (f->shard_mode < 0) return fail(FSM_EINVAL, "fsm_shard_map was not called");
  Opts o;
  int rc = resolve_opts(opts, &o);
  if (rc) return rc;
  if (!f->h_sh) {
    CUDA_TRY(cudaMallocHost(&f->h_sh, fsm_s::kRing * 8 * sizeof(uint32_t)));
    for (auto& e : f->sh_ev) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  const uint64_t seq = f->sh_next++;
  const uint32_t slot = (uint32_t)(seq % fsm_s::kRing);
  auto& sp = f->spend[slot];
  if (sp.active) CUDA_TRY(cudaEventSynchronize(f->sh_ev[slot]));  // ring wrapped
  sp = fsm_s::ShardPend{};
  sp.active = true;
  sp.seq = seq;
  sp.N = (f->shard_len + o.B - 1) / o.B;
  sp.scheme = f->shard_scheme;
  *ticket = seq;
  if (f->shard_mode != 3) {  // host fix-up modes: finish now
    sp.done = true;
    sp.rc = fsm_shard_finish(f, d_maps, G, rank, opts, d_chunk_ends_local, &sp.res);
    return FSM_OK;
  }
  const uint32_t nt = f->n + 1;
  if (!f->d_small) CUDA_TRY(cudaMalloc(&f->d_small, 64 * sizeof(uint32_t)));
  CUDA_TRY(launch_compose(reinterpret_cast<const uint8_t*>(d_maps), G, map_bytes_nt(nt), map_cnt_off(nt), f->img.q0t,
                          rank, f->d_small, o.st));
  ShardScratch S3;
  if ((rc = ensure_shard(f, &S3))) return rc;
  CUDA_TRY(cudaMemsetAsync(f->d_small + 5, 0, 4, o.st));
  if (d_chunk_ends_local && f->shard_len)
    CUDA_TRY(launch_fix_prefix_fused(S3.states, S3.cand, S3.info + 8, S3.grp, f->d_small, f->img.inv, f->n,
                                     d_chunk_ends_local, f->d_small + 5, o.st));
  CUDA_TRY(cudaMemcpyAsync(f->h_sh + slot * 8, f->d_small, 6 * sizeof(uint32_t), cudaMemcpyDeviceToHost, o.st));
  CUDA_TRY(cudaEventRecord(f->sh_ev[slot], o.st));
  sp.pipe_ticket = f->shard_ticket;  // the shard's pipeline run: collected by the wait
  f->shard_ticket = 0;
  return FSM_OK;
}

int fsm_shard_wait(fsm_t f, uint64_t ticket, fsm_result* out) {
  ApiScope api_scope_("fsm_shard_wait");
  if (!f || !out) return fail(FSM_EINVAL, "NULL handle/out");
  const uint32_t slot = (uint32_t)(ticket % fsm_s::kRing);
  auto& sp = f->spend[slot];
  if (!sp.active || sp.seq != ticket) return fail(FSM_EINVAL, "unknown or already collected shard ticket");
  sp.active = false;
  if (sp.done) {
    *out = sp.res;
    return sp.rc;
  }
  CUDA_TRY(cudaEventSynchronize(f->sh_ev[slot]));
  const uint32_t* h = f->h_sh + slot * 8;
  if (sp.pipe_ticket) {
    fsm_result rr;
    uint32_t ff;
    const int rc = run_collect(f, sp.pipe_ticket, &rr, &ff);  // complete: frees its ring slot
    if (rc) return rc;
  }
  if (h[2] == 3) {
    const int code = -(int)h[3];
    char msg[96];
    std::snprintf(msg, sizeof(msg), "fsm_shard_map failed on rank %u (%s)", h[4], fsm_strerror(code));
    return fail(code < 0 ? code : FSM_EINVAL, msg);
  }
  if (h[2] == 2) {
    f->shard_prefer_exact = true;
    return fail(FSM_EAGAIN, "a rank's speculative shard map was invalid: redo the step with fsm_run_sharded");
  }
  if (h[2] || h[5]) return fail(FSM_EINVAL, "a shard start state is outside its candidate set");
  std::memset(out, 0, sizeof(*out));
  out->nchunks = sp.N;
  out->scheme_used = sp.scheme;
  const uint32_t fin = h[1];
  if (fin == f->n) return fail(FSM_ESYMBOL, "input symbol >= nsyms");
  out->final_state = f->inv[fin];
  out->accept = f->accept[out->final_state];
  out->accept_count = (uint64_t)h[3] | ((uint64_t)h[4] << 32);
  return FSM_OK;
}

}  // extern "C"

namespace {

// FSM_SCHEME_AUTO: profile the stream itself (fsm_select_scheme spreads a long one).
int select_auto(fsm_t f, const uint8_t* d_in, uint64_t len, const fsm_run_opts* opts) {
  fsm_scheme pick;
  return fsm_select_scheme(f, d_in, len, opts, &pick, nullptr);
}

}  // namespace
