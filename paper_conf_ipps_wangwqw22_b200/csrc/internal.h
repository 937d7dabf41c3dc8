// internal.h — shared declarations of the sm_100a implementation behind
// include/gspec.h.  Nothing here is visible through the C ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "gspec.h"

namespace gspec {

// Table formats of the transformed DFA.
enum Mode : uint32_t {
  MODE_U8 = 1,   // raw-byte table, u8 codes, accept in bit 7, whole table in smem
  MODE_U16 = 2,  // classed table, u16 codes = tid | acc<<15, hot rows (tid < H) in smem
  MODE_U32 = 3,  // classed table, u32 codes = tid | acc<<31, hot rows in smem
  MODE_U16H = 4, // MODE_U16 with every row in smem: no hot test on the lookup path
  MODE_U16D = 5, // MODE_U16 whose cold rows are delta rows in smem: a hot base row + <= 2
                 // exceptions (8 B each); chosen only when every cold row compresses
};

constexpr uint32_t kDeltaExc = 2;        // exceptions per delta row
constexpr int MODE_U16D1 = 6;  // template-only: MODE_U16D image with delta_exc == 1 (the walk kernels' step)
constexpr uint32_t kInvalidMap = 0xFFFFFFFEu;  // map entry of a speculative shard map that must be redone
constexpr uint32_t kErrorMap = 0xFFFFFFFDu;    // map of a rank whose fsm_shard_map failed (count[0] = -status)
constexpr uint32_t kPendEnd = 0xFFFFFFFCu;     // end of a memoized helper record not walked yet (R28)
constexpr uint32_t kDeltaBaseMax = 8192;  // MODE_U16D: max shared-window offset of the staged table

constexpr uint32_t kQsMax = 16;     // QS cap ("top 16 states")
constexpr uint32_t kImgFull = 64;   // lookback > 2: pair images kept with multiplicities up to this size (R25)
constexpr uint32_t kLookbackMax = 16;
constexpr uint32_t kVrMax = 16;     // VR^end / VR^others slots
constexpr uint32_t kSlots = 2 * kVrMax;
constexpr uint32_t kEnumMax = 64;   // ENUM: transformed states incl. poison (maps of 32 or 64 entries)
constexpr uint32_t kEnumSmallMax = 32;  // ENUM in one launch (k_enum_small): 32-entry maps only

// POD device view of a loaded DFA, passed by value to every kernel.
struct DevImage {
  uint32_t mode;
  uint32_t n;       // real states; poison tid = n; nt = n + 1
  uint32_t nsyms;
  uint32_t C;       // byte classes (incl. the poison class when nsyms < 256)
  uint32_t H;       // hot rows in smem (MODE_U16/U32); all rows for MODE_U8
  uint32_t q0t;     // transformed start state
  uint32_t smem_table_bytes;  // bytes of the smem copy of the table
  // ENUM on small alphabets (nsyms <= 4, nt <= 64, MODE_U8): multi-symbol step table
  // TK[tid][combo] (walk.cuh; K = 8 symbols for nsyms <= 2, else 4) staged after the
  // table; nullptr when not built.  DESIGN.md §5.3.
  const uint32_t* TK;
  uint32_t tk_bytes;
  uint32_t tk_syms;  // K
  // K = 8 and nt <= 8: byte offset in the staged TK image of the packed-map
  // table PK[combo] (8 bytes: byte t = the tid after the 8 symbols from tid t | accepting states
  // among them << 4), so ONE lookup advances all 8 enumeration chains by 8 symbols; 0 = none
  uint32_t pk_off;
  const uint8_t* T8;          // MODE_U8: [256 codes][256 bytes] next code
  const uint16_t* T16;        // MODE_U16: [nt][C]
  const uint32_t* T32;        // MODE_U32: [nt][C]
  const uint8_t* cls;         // [256] byte -> class
  const uint8_t* cls2;        // MODE_U16H: [256] byte -> 2*class (staged instead of cls)
  const uint32_t* qs2;        // [C*C][kQsMax] ranked lookback candidates (tids)
  const uint8_t* qs2_len;     // [C*C]
  const uint32_t* qs2_img;    // [C*C] image size
  const uint32_t* tid2code;   // [nt]
  const uint32_t* code2tid;   // MODE_U8: [256]
  const uint32_t* inv;        // [nt] tid -> original id (poison -> n)
  const uint8_t* acc;         // [nt] accept by tid
  // MODE_U16D: the whole shared-memory table image
  //   [hot rows 0..H-1][poison row (= row H)][rows of the X tids][pad to 256][class map: 2*class,
  //   256 B][delta rows]
  // Codes are pre-multiplied: hot tid t < H -> t*C, poison -> H*C, X tid -> its slot*C (H+1..),
  // cold tid -> HC1 + its rank among the cold tids, accept flag in bit 15.  Delta row of a cold tid: x = (2*C*base tid) << 16 | e1 << 8 | e0
  // (e = 2*exception class, 0xFF = none; the row offset is made absolute at staging),
  // y = code0 | code1 << 16.
  const uint2* Dl;
  uint32_t delta_off;         // byte offset of the delta rows (16-aligned)
  uint32_t D;                 // delta rows (cold real tids)
  uint32_t cls_off;           // byte offset of the doubled class map (256-aligned)
  uint32_t HC1;               // (H + 1) * C (+ X * C): the first cold code
  // 1 when every delta row has at most one exception (e1 = 0xFF, y = code0): the hot set is then
  // the top-H tids plus the X tids that need two (hot slots H+1.., after the poison row), and the
  // walk kernels use the one-exception step; 2 otherwise
  uint32_t delta_exc;
};

// Global record store (hierarchical store, level 3).
// Slot s of chunk c lives at [s * cap + c]; END slots [0, vr_end), OTH slots
// [kVrMax, kVrMax + vr_oth).
struct RecStore {
  uint64_t cap;
  uint32_t* start;
  uint32_t* end;
  uint32_t* cnt;
  uint32_t* n_end;     // [cap] records ever appended to VR^end
  uint32_t* n_oth;     // [cap] records ever appended to VR^others
  uint32_t* oth_base;  // [cap] n_oth snapshot for this round's helpers
  uint8_t* next_qs;    // [cap] QS cursor
  uint32_t* ref_start; // [cap] immutable round-0 path (fusion reference)
  uint32_t* ref_end;
  uint32_t* ref_cnt;
  uint32_t* x;         // [cap+1] incoming state of chunk c (x[N] = final)
  uint32_t* cur_end;   // [cap] the chunk's current end (c.3: cur_end), constant during a verification
  uint8_t* found;      // [cap]
  // per-round scratch of the verify/recover kernel
  uint8_t* ulen;       // [cap] untried QS candidates of chunk c
  uint8_t* upos;       // [cap][kQsMax] their QS positions (phase T), for H2 and the cursor
  uint8_t* next_new;   // [cap] QS cursor after this round's helpers
  uint8_t* hcnt;       // [cap] helpers assigned to chunk c this round
  uint32_t* prefU;     // [cap] NF: exclusive prefix of ulen over c > f
  uint32_t* task_chunk;  // [cap+1] task slot -> chunk (0xFFFFFFFF = none)
  uint32_t* task_start;  // [cap+1]
  uint32_t* task_j;      // [cap+1] helper index within its chunk
  uint32_t* tstart;      // [cap] dense rounds: task start of chunk c, 0xFFFFFFFF = no task
  uint32_t* bflag;       // [cap / 32 + 1] fused round-0 verification: tile-boundary arrivals
  // fused round-0 verification counters {checks, matches, tasks, reread, ztot, ~first task
  // chunk (0 = none), moved, warps}: zero between runs (the last warp of a run clears them)
  unsigned long long* v0c;
};

// Device control block of the verify/recover kernel.
struct Ctl {
  uint64_t f;            // verified frontier
  uint32_t tf;           // t_f
  uint32_t pad0;
  uint64_t fmin;         // frontier candidate of this round
  uint32_t changed[4];   // Jacobi flags (rotating)
  uint32_t done;
  uint32_t status;
  uint64_t rounds;
  uint64_t tasks_mustdo, tasks_sre, tasks_helper, reread_bytes, verify_checks, verify_matches,
      active_sum;
  uint64_t accept_count;
  uint64_t nA, I, nU;    // nA: A-task entries of the task list handed to a dense round (the rest are helpers)
  uint64_t jacobi_iters;
  uint64_t ntask[2];     // [0]: length of the task list handed to a dense round; [1]: round-0 accept-count accumulator
  uint64_t it_fm[3], it_checks[3], it_matches[3], it_ntask[3];  // per relaxation pass (rotating)
  uint64_t it_reread[3];  // round-0 SRE pass with inline tasks: bytes re-walked (rotating)
  uint32_t dense_pending;  // verify exited: a dense task round (frontier fmin) must run first
  uint32_t nstamp;         // phase timestamps of the last verify launch (%globaltimer, ns)
  uint64_t stamp[24];
  uint32_t zdone;        // finalize tickets (the last CTA publishes the block to h_out)
  uint32_t xfin;         // transformed final state (written by the last kernel of a run)
  uint32_t pad1;
  // run timeline (%globaltimer ns; GSPEC_STAMPS=1): spec entry, last spec warp done,
  // verify entry (before table staging), verify exit (last CTA, before the host publish)
  uint64_t tl[4];
  // device-driven dense rounds (no host round trip): the verify finalize sets `finished`
  // (later launches of the run return at once); the finish kernel counts dense rounds;
  // `dense_denied` = a verify launch ran a dense round in-kernel because the run had no
  // task-kernel slot left (the host raises its slot count for the next run)
  uint32_t finished, dense_rounds, dense_denied, pad2;
  // FSM_SCHEME_PM_TREE (pm_tree.cu): stage-1 lookups, entries marked invalid, stage-2 jumps
  uint64_t pm_merge_checks, pm_invalid_marks, pm_jumps;
  uint64_t helper_walks;  // RR / NF helper records actually walked (memoized helpers, R28)
  uint64_t walked_bytes;  // bytes the dense-round task kernels actually walked (R30 early exit)
  uint32_t segn[3];       // checkpointed dense round: chains appended by pass p in segn[p % 3] (R30)
  uint32_t seg_done;      // R30 last pass: warps done (the last one commits the round; reset by it)
};

struct RunParams {
  const uint8_t* in;
  uint32_t q0t;    // transformed start state of chunk 0 (q0 of the DFA, or a shard candidate)
  uint64_t len;
  uint32_t B;
  uint64_t N;
  int scheme;
  uint32_t k;      // paths per chunk in round 0
  uint32_t qs_cap;
  uint32_t vr_end, vr_oth;
  uint32_t dense;  // 1: hand rounds with many SRE tasks to the TMA task kernel (verify exits)
  uint32_t dense_slots;  // task-kernel launches still queued behind this verify launch
  Ctl* ctl_init;   // non-null: the first spec kernel initialises this control block (no H2D copy)
  const uint32_t* q0_dev;  // non-null: chunk 0's start is read from the device (shard candidates)
  Ctl* h_out;      // non-null: pinned host slot; the finalize step writes the control block there
  uint32_t stamps; // 1: record the run timeline (Ctl::tl), profiling only
  const uint32_t* qsc;     // non-null: per-chunk QS [N][kQsMax] of a lookback > 2 (k_qs_long)
  const uint8_t* qsc_len;  // [N]
  // fused round-0 verification (SRE, spec-1, accurate speculation): the TMA spec kernel
  // checks every chunk against its predecessor's round-0 end as its tiles finish, runs the
  // mismatches' recoveries inline and, when no recovery changed an end, completes the run
  uint32_t v0;             // 1: fused (v0_ctl, v0_bflag set)
  Ctl* v0_ctl;
  uint32_t* v0_bflag;      // [tiles] tile-boundary arrival counters (+2 per run, never reset)
  uint32_t* v0_chunk_ends; // nullable: the run's chunk ends (original ids)
  uint32_t tma_evict_normal;  // 1: input TMA loads with L2 evict_normal (else evict_first)
  uint32_t lazy_helpers;      // 1: RR / NF helper records are memoized (walked when first matched, R28)
  // checkpointed dense rounds (R30): the round-0 TMA walk stores {code, count so far}
  // of its path every 2^ck_shift bytes at ck[j * N + c] (j = bytes / 2^ck_shift - 1); a dense
  // task stops at the first checkpoint where it meets that path.  ck_shift 0 = off.
  uint2* ck;
  uint32_t ck_shift;
  uint32_t ck_seg;  // bytes per segment pass of a checkpointed dense round (0: plain task kernel)
  void* ck_list;    // the passes' two lists of running chains, [2][rs.cap] x 16 B
};

// GSPEC_STAMPS=1: kernels record the run timeline in Ctl::tl (one extra atomic per warp).
inline bool stamps_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_STAMPS");
    v = e ? atoi(e) : 0;
  }
  return v != 0;
}

// Programmatic dependent launch (PDL) between the two kernels of a run and
// between consecutive runs: the next kernel is launched while the previous one
// drains and waits in griddepcontrol.wait (after its table staging) for the
// previous grid's completion and memory flush.  Opt-in (GSPEC_PDL=1): measured on
// c2 it does not shorten the step (0.3237 vs 0.3232 ms) — the verify CTAs cannot
// become resident before the spec CTAs (full shared memory) exit.
// Fused round-0 verification in the spec kernel (RunParams::v0): opt-in, GSPEC_V0=1.
// Measured neutral on C2 (spec kernel +16 us, verify launch -16 us: 3446 vs 3447 GB/s) and
// slightly slower on C4 (3.34 vs 3.29 ms: the per-tile epilogue competes with the walk for
// issue and LSU slots), so the separate verify kernel stays the default.
inline bool v0_disabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_V0");
    v = (e && atoi(e) == 1) ? 0 : 1;
  }
  return v != 0;
}

// TMA input L2 promotion (GSPEC_TMA_PROMO: 0 = 256 B default, 1 = 64 B, 2 = none) and the
// input's L2 eviction policy (GSPEC_TMA_EVICT: 0 = evict_first default, 1 = evict_normal)
inline int tma_promotion() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_TMA_PROMO");
    v = e ? atoi(e) : 0;
  }
  return v;
}

// R30 checkpoint interval of dense rounds (GSPEC_CK: bytes, a power of two >= 64; 0 = off,
// the plain TMA task kernel).  Returns log2 of the interval, 0 when off.
inline uint32_t ck_shift_default() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_CK");
    const long b = e ? atol(e) : 512;
    v = 0;
    if (b >= 64 && (b & (b - 1)) == 0)
      while ((1l << v) < b) v++;
  }
  return (uint32_t)v;
}

// R30 segment of a checkpointed dense-round pass (GSPEC_CK_SEG: bytes, a multiple of the
// checkpoint interval; default a quarter of the chunk rounded up to the interval).
inline uint32_t ck_seg_for(uint32_t B, uint32_t ck_shift) {
  static long v = -2;
  if (v == -2) {
    const char* e = getenv("GSPEC_CK_SEG");
    v = e ? atol(e) : -1;
  }
  const uint32_t cp = 1u << ck_shift;
  uint32_t seg = v > 0 ? (uint32_t)v : (B / 4 + cp - 1) / cp * cp;
  seg = (seg + cp - 1) / cp * cp;
  return seg < cp ? cp : seg;
}

// GSPEC_TK_PK=0: enumeration on small alphabets without the packed-map table (A/B; read at
// every fsm_load)
inline bool tk_pk_disabled() {
  const char* e = getenv("GSPEC_TK_PK");
  return e && atoi(e) == 0;
}

inline int tma_evict_mode() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_TMA_EVICT");
    v = e ? atoi(e) : 0;
  }
  return v;
}

// RR / NF helpers memoized (R28): opt-in, GSPEC_LAZY_HELPERS=1.  Measured slower on C3
// (RR 3.14 vs 2.53 ms, NF 8.56 vs 2.45 ms): the helpers the verification does consult sit
// on its critical path, and walking them there, one per owner thread and pass, costs more
// than walking every helper up front on the TMA task kernel.
inline bool lazy_helpers_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_LAZY_HELPERS");
    v = (e && atoi(e) == 1) ? 1 : 0;
  }
  return v != 0;
}

inline bool pdl_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_PDL");
    v = e ? atoi(e) : 0;
  }
  return v != 0;
}

// Host-side launch-config cache: raises the kernel's dynamic-smem limit
// (monotonically, so concurrent handles with different tables never lower it
// under each other) and queries occupancy once per (kernel, smem, block).
inline cudaError_t kernel_setup(const void* kern, uint32_t smem, int block, int* occ) {
  struct Key {
    const void* k; uint32_t smem; int block;
    bool operator<(const Key& o) const {
      return k != o.k ? k < o.k : smem != o.smem ? smem < o.smem : block < o.block;
    }
  };
  static std::mutex mu;
  static std::map<Key, int> occ_cache;
  static std::map<const void*, uint32_t> smem_max;
  std::lock_guard<std::mutex> g(mu);
  static int optin = -1;  // probing callers ask for sizes that may not fit: refuse those without
  if (optin < 0) {        // an API error (a failed attribute call would leave a stale last error)
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) optin = 0;
  }
  if (optin > 0 && smem > (uint32_t)optin) return cudaErrorInvalidValue;
  uint32_t& mx = smem_max[kern];
  if (smem > mx) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) {
      (void)cudaGetLastError();
      return e;
    }
    mx = smem;
  }
  const Key key{kern, smem, block};
  auto it = occ_cache.find(key);
  if (it == occ_cache.end()) {
    int o = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kern, block, smem);
    if (e != cudaSuccess) {
      (void)cudaGetLastError();
      return e;
    }
    it = occ_cache.emplace(key, o).first;
  }
  if (occ) *occ = it->second;
  return cudaSuccess;
}

// GSPEC_TK=0: the enumerative walk ignores the multi-symbol table (A/B; tests compare both)
inline bool tk_disabled() {
  const char* e = getenv("GSPEC_TK");
  return e && e[0] == '0';
}

inline int device_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  return sms;
}

// ---- launchers (each returns the cudaError_t of the launch) ------------------
cudaError_t launch_build_qs2_raw(const uint32_t* d_ttc, uint32_t n, uint32_t C, uint32_t* scratch, uint32_t grid,
                                 uint32_t* qs2, uint8_t* qs2_len, uint32_t* qs2_img, cudaStream_t st);
// *tma_done (nullable): chunks the TMA spec kernel walked (the rest went to the generic kernel)
cudaError_t launch_spec_exec(const DevImage& img, const RunParams& rp, const RecStore& rs, cudaStream_t st,
                             uint64_t* tma_done = nullptr);
cudaError_t launch_spec_tma(const DevImage& img, const RunParams& rp, const RecStore& rs, int sms, cudaStream_t st,
                            uint64_t* n_done);
// Dense recovery round, device-driven: if the preceding verify launch left a dense round
// pending (ctl->dense_pending), its task list (rs.task_chunk/task_start, ctl->ntask[0]
// entries, all chunks >= ctl->fmin) is re-walked by the TMA-gather task kernel (full
// chunks) and the finish kernel (tail chunk, round commit); otherwise both return at once.
// Enqueued without any host synchronisation.
cudaError_t launch_task_dense(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* ctl, int sms,
                              cudaStream_t st);
// Paper-literal SRE: one CTA, one thread per chunk (N <= literal_max_chunks()),
// Alg. 2 L2-6 + Alg. 3 verbatim; results and stats in *ctl (zeroed by the caller).
// FSM-level batching: one CTA per (DFA, stream) pair of one table format.
cudaError_t launch_multi(int mode, const DevImage* d_imgs, const uint8_t* const* d_ins, const uint64_t* d_lens,
                         const uint32_t* d_pairs, uint32_t npairs, uint32_t smem, uint32_t B, uint32_t* d_fin,
                         unsigned long long* d_cnt, unsigned long long* d_stats, cudaStream_t st);
uint32_t literal_max_chunks();
cudaError_t launch_literal_sre(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* ctl,
                               uint32_t* d_chunk_ends, cudaStream_t st);
bool spec_path_generic_only();  // GSPEC_SPEC_PATH=generic forces the non-TMA kernel (A/B tests)
cudaError_t launch_verify_recover(const DevImage& img, const RunParams& rp, const RecStore& rs, Ctl* d_ctl,
                                  uint64_t* d_block_tmp, uint32_t* d_chunk_ends, cudaStream_t st, int sm_count);
uint64_t enum_scratch_bytes(uint64_t nsub);
// ENUM of a small stream (nsub <= enum_small_max_sub() sub-chunks) in ONE launch
uint64_t enum_small_max_sub();
uint64_t enum_small_scratch_bytes(uint64_t nsub);
cudaError_t launch_enum_small(const DevImage& img, const RunParams& rp, uint32_t E, void* scratch, uint32_t* ticket,
                              uint32_t* d_chunk_ends, Ctl* d_ctl, cudaStream_t st);
cudaError_t launch_enum_full(const DevImage& img, const RunParams& rp, uint32_t E, void* scratch,
                             uint32_t* d_chunk_ends, Ctl* d_ctl, uint32_t* d_x_final, cudaStream_t st, int sms,
                             int phases = 3, const uint8_t** top_M = nullptr, const uint64_t** top_C = nullptr);
cudaError_t launch_features_raw(const DevImage& img, const uint32_t* d_ttc, const uint8_t* in, uint64_t len,
                                uint32_t B, uint64_t N, const uint32_t* d_x, uint32_t k, uint32_t qs_cap,
                                unsigned long long* d_counts, uint32_t* d_seen, unsigned long long* d_uniq,
                                cudaStream_t st);

uint64_t batch_totals_bytes();
cudaError_t launch_batch(const DevImage& img, const uint8_t* in, const uint64_t* off, const uint64_t* cbase,
                         uint32_t ns, uint64_t N, uint32_t B, uint32_t* cs, uint32_t* rs, uint32_t* re, uint32_t* rc,
                         uint32_t* fin,
                         unsigned long long* count, uint32_t* chunk_ends, void* tot, cudaStream_t st, int sms);

cudaError_t launch_shard_image(const DevImage& img, const uint32_t* ttc, const uint8_t* w, uint32_t L, uint32_t* mark,
                               uint32_t* list, uint32_t* count, cudaStream_t st);
cudaError_t launch_shard_fuse(const DevImage& img, const uint8_t* in, uint64_t len, uint32_t B, const uint32_t* cand,
                              uint32_t ncand, uint32_t max_chunks, uint32_t* states, unsigned long long* cnt,
                              uint32_t* info, cudaStream_t st);
cudaError_t launch_map_init(uint32_t* mend, unsigned long long* mcnt, uint32_t nt, cudaStream_t st);
cudaError_t launch_shard_fuse_ref(const DevImage& img, const uint8_t* in, uint64_t len, uint32_t B,
                                  const uint32_t* cand, const uint32_t* ncand_p, uint32_t max_chunks, uint32_t* states,
                                  uint32_t* merged, long long* dcnt, uint32_t* unmerged, cudaStream_t st);
cudaError_t launch_map_fused(const uint32_t* cand, const uint32_t* ncand_p, const long long* dcnt, const uint32_t* fin_p,
                             const unsigned long long* count_p, uint32_t* mend, unsigned long long* mcnt,
                             const uint32_t* unmerged, cudaStream_t st);
cudaError_t launch_fix_prefix_fused(const uint32_t* states, const uint32_t* cand, const uint32_t* ncand_p,
                                    const uint32_t* merged, const uint32_t* srank_p, const uint32_t* inv,
                                    uint32_t poison, uint32_t* chunk_ends, uint32_t* err, cudaStream_t st);
cudaError_t launch_build_img2_raw(const uint32_t* d_ttc, uint32_t n, uint32_t C, uint32_t* scratch, uint32_t grid,
                                  uint32_t* img_s, uint32_t* img_m, uint8_t* img_n, cudaStream_t st);
cudaError_t launch_qs_long(const DevImage& img, const uint32_t* d_ttc, const uint8_t* in, uint32_t B, uint64_t N,
                           uint32_t L, const uint32_t* img_s, const uint32_t* img_m, const uint8_t* img_n,
                           uint32_t* qsc, uint8_t* qsc_len, int sms, cudaStream_t st);
uint64_t pm_tree_scratch_bytes(uint64_t N, uint32_t k, uint32_t* levels);
cudaError_t launch_pm_tree(const DevImage& img, const RunParams& rp, const RecStore& rs, uint32_t k, void* scratch,
                           Ctl* ctl, uint32_t* d_chunk_ends, int sms, cudaStream_t st, uint32_t* launches);
cudaError_t launch_feat_conv(const DevImage& img, const uint32_t* d_ttc, const uint8_t* in, uint32_t nwin,
                             uint32_t wmax, uint32_t* d_out, cudaStream_t st);
cudaError_t launch_map_fused_publish(const uint32_t* cand, const uint32_t* ncand_p, const long long* dcnt,
                                     const uint32_t* fin_p, const unsigned long long* count_p, uint32_t* mend,
                                     unsigned long long* mcnt, const uint32_t* unmerged, uint64_t mapb,
                                     uint8_t* const* peers, uint32_t G, uint32_t rank, uint32_t set,
                                     unsigned long long seq, cudaStream_t st);
cudaError_t launch_publish(const uint8_t* own_map, uint64_t mapb, uint8_t* const* peers, uint32_t G, uint32_t rank,
                           uint32_t set, unsigned long long seq, cudaStream_t st);
cudaError_t launch_map_error(uint32_t* mend, unsigned long long* mcnt, uint32_t nt, uint32_t code, cudaStream_t st);
cudaError_t launch_set_u32(uint32_t* p, uint32_t v, uint32_t* p2, uint32_t v2, cudaStream_t st);
cudaError_t launch_map_write(const uint32_t* cand, uint32_t ncand, const uint32_t* grp,
                             const unsigned long long* prefix, const uint32_t* pfinal, const unsigned long long* pcount,
                             uint32_t* mend, unsigned long long* mcnt, cudaStream_t st);
cudaError_t launch_map_enum(const uint8_t* topM, const unsigned long long* topC, uint32_t nt, uint32_t* mend,
                            unsigned long long* mcnt, cudaStream_t st);
cudaError_t launch_compose(const uint8_t* maps, uint32_t G, uint64_t map_bytes, uint64_t cnt_off, uint32_t q0t,
                           uint32_t rank, uint32_t* out, cudaStream_t st,
                           const unsigned long long* wflags = nullptr, unsigned long long seq = 0,
                           uint32_t* wstatus = nullptr);
cudaError_t launch_fix_prefix(const uint32_t* states, uint32_t ncand, uint32_t ci, uint32_t nj, const uint32_t* inv,
                              uint32_t* chunk_ends, cudaStream_t st);

// ---- handle ------------------------------------------------------------------
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
};

}  // namespace gspec

struct fsm_s {
  uint32_t n, nsyms, q0;
  std::vector<uint32_t> table;  // original table (host copy)
  std::vector<uint8_t> accept;
  std::vector<uint32_t> perm, inv;  // [n+1]
  std::vector<uint64_t> freq;       // [n]
  std::vector<uint8_t> cls;         // [256]
  gspec::DevImage img{};
  std::vector<void*> owned;         // device allocations of the image
  // scratch for runs (grown on demand)
  gspec::RecStore rs{};
  uint64_t rs_cap = 0;
  uint32_t rs_slots_alloc = 0;
  void* rs_base = nullptr;
  gspec::Ctl* d_ctl = nullptr;
  // in-flight runs: pinned Ctl mirrors (init + readback) and events per ring slot
  static constexpr uint32_t kRing = 32;
  gspec::Ctl* h_ctl = nullptr;        // pinned [kRing]
  cudaEvent_t ev[kRing][4] = {};      // start, after spec, after verify, after readback
  struct Pending {
    uint64_t seq = 0, N = 0;
    fsm_scheme scheme = FSM_SCHEME_SRE;
    uint32_t q0t = 0;
    bool active = false;
    uint32_t done_ev = 3;  // event that marks the result readable (2: zero-copy result)
    uint32_t launches = 0; // kernels enqueued for this run
    uint32_t dense_slots = 0;  // dense task-kernel slots queued for this run
    bool dense = false;        // dense rounds were enabled for this run
  } pend[kRing];
  uint64_t next_seq = 1;
  uint64_t* d_block_tmp = nullptr;
  size_t block_tmp_elems = 0;
  void* enum_base = nullptr;
  size_t enum_bytes = 0;
  void* feat_base = nullptr;
  size_t feat_bytes = 0;
  int sm_count = 0;
  int device = 0;
  fsm_scheme auto_scheme = FSM_SCHEME_SRE;
  double acc1_hint = 0.0;            // spec-1 accuracy from the selector's profile (dense-round gate)
  double conv_hint = 1.0;            // profile's fraction of windows converged within 16 KiB (R30 gate; 1 = unknown)
  uint32_t dense_hint = 4;           // task-kernel slots queued per dense run (dense rounds last seen)
  bool shard_prefer_exact = false;   // a speculative shard map was invalid once: use the exact map
  uint32_t* enum_ticket = nullptr;   // single-launch ENUM: finished-CTA counter (zeroed once)
  bool auto_selected = false;
  const uint32_t* d_ttc = nullptr;   // [nt][C] transformed tid x class table (prep/features)
  uint32_t* d_small = nullptr;       // small device scratch (ENUM final state, shard compose)
  // fsm_run_host staging
  void* h_dev_in = nullptr;
  void* h_dev_ce = nullptr;
  uint64_t h_in_cap = 0, h_ce_cap = 0;
  // sharded runs (state kept between fsm_shard_map and fsm_shard_finish)
  void* shard_base = nullptr;   // device scratch of the shard steps
  size_t shard_bytes = 0;
  int shard_mode = -1;          // 0 fused/single path, 1 enum, 2 multi-path, 3 fused with cand[0], 4 map failed
  uint64_t shard_ticket = 0;
  // asynchronous sharded steps (fsm_shard_finish_async / fsm_shard_wait): a ring of
  // pending finishes, their result words in pinned memory
  struct ShardPend {
    bool active = false;
    uint64_t seq = 0, N = 0, pipe_ticket = 0;
    fsm_scheme scheme = FSM_SCHEME_AUTO;
    bool done = false;       // finished synchronously (host fix-up modes): res/rc hold the outcome
    int rc = 0;
    fsm_result res{};
  } spend[kRing];
  uint32_t* h_sh = nullptr;              // pinned [kRing][8] result words of async finishes
  cudaEvent_t sh_ev[kRing] = {};
  uint64_t sh_next = 1;
  uint32_t last_nstamp = 0;            // verify phase timestamps of the last collected run
  uint64_t last_stamp[24] = {};
  uint64_t last_tl[4] = {};             // run timeline of the last collected run (GSPEC_STAMPS=1)
  void* batch_base = nullptr;            // fsm_run_batch scratch (offsets, chunk bases, records, totals)
  size_t batch_bytes = 0;
  cudaEvent_t batch_ev[2] = {nullptr, nullptr};
  uint8_t* prof_buf = nullptr;           // FSM_SCHEME_AUTO's spread 1 MiB profile sample
  // set by fsm_run_sharded_p2p around its fsm_shard_map call: the fused-mode map kernel then
  // also publishes the map to the peers (k_map_fused_publish) and sets p2p_published
  struct P2PPub {
    uint64_t mapb;
    uint8_t* const* peers;
    uint32_t G, rank, set;
    unsigned long long seq;
  };
  const P2PPub* p2p_pub = nullptr;
  // set by fsm_run_sharded_p2p around its fsm_shard_finish call: the composition kernel first
  // waits for the peers' arrival flags of this step (k_compose's wflags), no separate wait kernel
  struct P2PWait {
    const unsigned long long* flags;  // this step's G flags in the own mailbox
    unsigned long long seq;
    uint32_t* status;
  };
  const P2PWait* p2p_wait = nullptr;
  bool p2p_published = false;
  void* img2_base = nullptr;             // lookback > 2: full pair images (built at first use)
  uint32_t *img2_s = nullptr, *img2_m = nullptr;
  uint8_t* img2_n = nullptr;
  void* qsc_base = nullptr;              // lookback > 2: per-run QS table [N][kQsMax] + lengths
  uint64_t qsc_cap = 0;
  void* pm_base = nullptr;               // FSM_SCHEME_PM_TREE scratch (level maps, jump list)
  size_t pm_bytes = 0;
  void* ck_base = nullptr;               // R30: round-0 path checkpoints [B / 2^ck_shift - 1][N]
  size_t ck_bytes = 0;
  void* multi_base = nullptr;            // fsm_run_multi scratch when this handle is fsms[0] (its device)
  size_t multi_cap = 0;
  cudaEvent_t multi_ev[2] = {nullptr, nullptr};
  const uint8_t* shard_in = nullptr;
  uint64_t shard_len = 0;
  uint32_t shard_ncand = 0, shard_nj = 0;  // candidates; chunks covered by the fused prefix
  uint32_t shard_E = 0;
  fsm_scheme shard_scheme = FSM_SCHEME_SRE;
  std::vector<uint32_t> shard_cand, shard_grp, shard_dist;
};
