/* gspec.h — C ABI of the B200-native GSpecPal hot path (speculative
 * chunk-parallel DFA execution).
 *
 * Paper: Wang, Watling, Qiu, Wang, "GSpecPal: Speculation-Centric Finite State
 * Machine Parallelization on GPUs" (IPDPS'22).  "P:n" below cites line n of
 * /root/reference/PAPER.md; DESIGN.md restates every reading.
 *
 * The problem the ABI solves (Alg. 1): run a DFA (Q, Σ, q0, δ, F)
 * over one input stream; report the end state's accept/reject decision (the
 * output function φ is void) plus, reading R3, the number
 * of accepting positions and the state at the end of every chunk of
 * `chunk_bytes` bytes.  Every scheme returns exactly the sequential result;
 * speculation only changes the cost.
 *
 * Conventions (all entry points):
 *  - return 0 (FSM_OK) or a negative fsm_status; on error out-params are not
 *    written and fsm_last_error() holds a thread-local message;
 *  - every state id crossing the ABI is an ORIGINAL id (the frequency
 *    renumbering of P:319-330 is internal to the handle);
 *  - pointers named d_* are DEVICE pointers (e.g. torch CUDA tensors'
 *    data_ptr()), h_* are host pointers; both are borrowed for the call only;
 *  - all device work is enqueued on opts->stream (NULL = legacy default
 *    stream); the calls are synchronous: they synchronize that stream before
 *    filling host results;
 *  - a handle is not re-entrant: use one handle per concurrent stream.
 */
#ifndef GSPEC_H
#define GSPEC_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  FSM_OK = 0,
  FSM_EINVAL = -1,       /* invalid argument (see each call)                   */
  FSM_ENOMEM = -2,       /* device or host allocation failed                   */
  FSM_ECUDA = -3,        /* CUDA runtime error (message in fsm_last_error)     */
  FSM_ESYMBOL = -4,      /* an input byte >= nsyms (reading R4); outputs unset  */
  FSM_ENCCL = -5,        /* collective failed                                  */
  FSM_EUNSUPPORTED = -6, /* e.g. ENUM on a DFA with > 63 states                */
  FSM_EAGAIN = -7        /* fsm_shard_finish: a rank's speculative shard map was
                            invalid; every rank redoes fsm_shard_map_exact + the
                            exchange + fsm_shard_finish (all ranks see the same maps) */
} fsm_status;

/* Parallelization schemes (PM, SRE; P:195 RR; P:222 NF; P:89 ENUM). */
typedef enum {
  FSM_SCHEME_AUTO = 0, /* the decision-tree selector, cached per handle   */
  FSM_SCHEME_SEQ = 1,  /* Alg. 2: spec-1 + sequential verification/recovery      */
  FSM_SCHEME_PM = 2,   /* spec-k + parallel verification, must-do recoveries only */
  FSM_SCHEME_SRE = 3,  /* Alg. 3: recovery activated by the predecessor's end    */
  FSM_SCHEME_RR = 4,   /* Alg. 4: SRE + round-robin helpers over QS              */
  FSM_SCHEME_NF = 5,   /* Alg. 5: SRE + nearest-first helpers over QS            */
  FSM_SCHEME_ENUM = 6, /* enumerative: all-state chunk maps + composition scan  */
  FSM_SCHEME_CSE = 7,  /* convergence-set enumeration (P:300, P:427 [21][24]):
                          round 0 walks every lookback-2 candidate of each chunk up to
                          spec_k (default 8) — the whole image, which contains the true
                          start, whenever it has <= spec_k states — with path fusion
                          (paths that meet are walked once); SRE rounds recover what a
                          capped image missed.  Not chosen by FSM_SCHEME_AUTO. */
  FSM_SCHEME_PM_TREE = 8 /* faithful PM as published (Xia et al.; Fig. 2, Eq. 2
                          P:266-268): spec-k, ceil(log2 N) rounds of parallel
                          tree-like merging of k-entry chunk maps where a mismatch marks
                          the path invalid (delayed recovery), then a sequential stage from
                          q0 over the merged segments that recovers a chunk at once when
                          its incoming state has no valid record.  The paper's comparison
                          baseline (Fig. 8 "PM spec-4"); FSM_SCHEME_PM is the B200 reading
                          R17 chosen by the selector.  Not chosen by FSM_SCHEME_AUTO. */
} fsm_scheme;

typedef struct fsm_s* fsm_t;

typedef struct {
  uint32_t freq_policy;          /* 0 = static in-degree (Fig. 4), 1 = profile visits */
  const uint8_t* profile_sample; /* host bytes (read during the call only): freq_policy 1
                                    ranks states by their visits on it; with any policy the
                                    u8 format also places table rows bank-aware from it
                                    (layout only, results unchanged); NULL = no profile    */
  uint64_t profile_len;
  uint32_t smem_budget_bytes;    /* hot-row budget in shared memory; 0 = auto        */
  uint32_t force_mode;           /* 0 auto; 1 u8 raw-byte table; 2 u16 classed (hot rows in smem,
                                    cold rows in L2); 3 u32 classed; 4 u16 classed whose cold rows
                                    are delta rows in smem (hot base row + <= 2 exceptions, rows that
                                    do not compress stay in L2).  Auto picks 4 over 2 when the delta
                                    rows keep more frequency mass on chip. */
} fsm_load_opts;

typedef struct {
  fsm_scheme scheme;    /* FSM_SCHEME_*                                                  */
  uint32_t chunk_bytes; /* B: chunk c = [cB, min(len,(c+1)B)); multiple of 16; 0 = 4096   */
  uint32_t spec_k;      /* paths per chunk: PM (4) / CSE (8); 1..16; 0 = default   */
  uint32_t lookback;    /* lookback symbols L (2); 2..16 (reading R25); 0 = 2     */
  uint32_t qs_cap;      /* K: ranked candidates kept per chunk (16); 1..16; 0 = 16 */
  uint32_t vr_end;      /* VR^end slots per chunk (16); 1..16; 0 = 16              */
  uint32_t vr_others;   /* VR^others slots per chunk (16); 1..16; 0 = 16           */
  void* stream;         /* cudaStream_t                                                   */
} fsm_run_opts;

typedef struct {
  uint32_t final_state;      /* original id of the state after the last symbol        */
  uint32_t accept;           /* F contains final_state                          */
  uint64_t accept_count;     /* #positions i in [1,len] whose state is accepting (R3)  */
  uint64_t nchunks;          /* ceil(len / chunk_bytes)                                */
  fsm_scheme scheme_used;
  uint32_t rounds;           /* verification/recovery rounds with a must-do task       */
  uint64_t tasks_total, tasks_mustdo, tasks_sre, tasks_helper;
  uint64_t reread_bytes;     /* bytes re-walked by recovery tasks (nominal chunk bytes) */
  uint64_t verify_checks, verify_matches; /* runtime speculation accuracy    */
  double avg_active_workers; /* mean active workers per round (Table III analogue)    */
  double ms_spec, ms_verify; /* device time of speculative execution / verify+recover */
  uint32_t kernel_launches;  /* kernels this run launched (spec, verify, dense rounds, ENUM levels) */
  /* FSM_SCHEME_PM_TREE only (0 otherwise): stage-1 entry lookups, entries marked invalid
   * (delayed recoveries), stage-2 segments taken through their merged maps.  For that
   * scheme rounds = merge rounds, tasks_mustdo = stage-2 recoveries, verify_checks =
   * stage-2 steps, verify_matches = stage-2 jumps. */
  uint64_t pm_merge_checks, pm_invalid_marks, pm_jumps;
  /* RR / NF with memoized helpers (opt-in GSPEC_LAZY_HELPERS=1, R28): helper
   * records actually walked (a helper's record then holds its start at once and is walked
   * when a verification first matches it); 0 with eager helpers.  tasks_helper and
   * reread_bytes count every assigned helper either way, as the round semantics define. */
  uint64_t helper_walks;
  /* Bytes the dense-round task kernels actually walked (R30: a task stops where
   * its path meets the chunk's round-0 path at a checkpoint, so this is at most
   * reread_bytes' share of those rounds); diagnostic, 0 when no dense round ran. */
  uint64_t task_walked_bytes;
} fsm_result;

typedef struct {
  double acc1;              /* spec-1 accuracy on the sample (Table II)         */
  double acck;              /* spec-k accuracy (k = opts->spec_k)                      */
  double input_sensitivity; /* max-min of per-segment acc1 over 8 segments (R19)       */
  double uniq10;            /* mean #unique states after 10 transitions from all */
  uint32_t nstates;
  /* Granularity (reading R29): windows every 4 KiB of the profile, each
   * walking every state of its lookback-2 image until all paths are in one state
   * (checked every 64 B, up to 16 KiB).  conv{4,8,16}k = fraction of windows converged
   * within that many bytes; chunk_bytes = the smallest of 4/8/16 KiB with a fraction
   * >= 3/4 that still leaves >= SMs x 768 chunks of the stream (len as passed), else
   * 4096.  A recommendation: fsm_run uses opts->chunk_bytes as given. */
  uint32_t chunk_bytes;
  double conv4k, conv8k, conv16k;
} fsm_features;

/* Load a DFA.  table: host uint32 [nstates][nsyms], row-major, original ids;
 * accept: host uint8 [nstates] (0/1); start < nstates.  Both are COPIED.
 * Builds the frequency-transformed device image, byte classes, the
 * lookback pair table on the device.  Errors: FSM_EINVAL if nstates = 0,
 * nsyms not in [1,256], start >= nstates, an entry >= nstates or NULL arrays;
 * FSM_EUNSUPPORTED if nstates >= 2^24. */
int fsm_load(const uint32_t* table, uint32_t nstates, uint32_t nsyms, uint32_t start,
             const uint8_t* accept, const fsm_load_opts* opts, fsm_t* out);

/* Number of chunks = ceil(len / chunk_bytes) (chunk_bytes 0 means 4096). */
uint64_t fsm_num_chunks(uint64_t len, uint32_t chunk_bytes);

/* Run the DFA over device bytes d_input[0..len) (reading R2 for the
 * partition).  d_chunk_ends (device, nullable) receives nchunks uint32 original
 * ids: the state after each chunk's last symbol.  opts nullable (defaults).
 * Errors: FSM_EINVAL (bad opts, NULL input with len > 0), FSM_ESYMBOL (an input
 * byte >= nsyms; detected through the absorbing poison state), FSM_ENOMEM,
 * FSM_ECUDA, FSM_EUNSUPPORTED (ENUM with nstates > 63). */
int fsm_run(fsm_t fsm, const uint8_t* d_input, uint64_t len, const fsm_run_opts* opts,
            uint32_t* d_chunk_ends, fsm_result* out);

/* Asynchronous fsm_run: enqueues the whole run (kernels + the small result
 * readback into pinned memory) on opts->stream and returns a ticket at once;
 * fsm_wait(ticket) blocks until that run is done and fills *out.  Up to 32
 * runs may be in flight per handle (they execute in stream order and reuse
 * the handle's scratch one after another).  d_input/d_chunk_ends must stay
 * valid until the run completes.  With FSM_SCHEME_AUTO the first call may
 * synchronously profile the input (selector). */
int fsm_run_async(fsm_t fsm, const uint8_t* d_input, uint64_t len, const fsm_run_opts* opts,
                  uint32_t* d_chunk_ends, uint64_t* ticket);
int fsm_wait(fsm_t fsm, uint64_t ticket, fsm_result* out);

/* ---- stream-level batching (Alg. 1 L2-3) ------------------------
 * Runs the DFA over nstreams independent streams, stream s = d_input[h_offsets[s]
 * .. h_offsets[s+1]) (host array of nstreams+1 non-decreasing byte offsets; any
 * alignment; empty streams allowed).  Each stream is split into chunks of
 * opts->chunk_bytes (its last chunk may be short); its first chunk starts at q0,
 * the others at the lookback-2 prediction; one thread per stream then
 * verifies its chain and re-executes each mispredicted chunk from the verified
 * state (Alg. 2 L7-11, with path fusion).  Outputs (device, caller-owned):
 * d_final[s] (uint32 original id; == nstates marks a stream with a byte >= nsyms),
 * d_count[s] (uint64 accept count, R3), d_chunk_ends (nullable; uint32 per chunk,
 * streams' chunks in order, fsm_batch_chunks() entries).  Synchronous; returns
 * FSM_ESYMBOL (outputs still written) if any stream saw an invalid byte. */
typedef struct {
  uint64_t nstreams, nchunks;
  uint64_t recoveries;       /* mispredicted chunks re-executed (== chunks whose lookback
                                prediction differs from the true start state)           */
  uint64_t reread_bytes;     /* bytes those recoveries covered (nominal)                 */
  uint64_t invalid_streams;  /* streams that saw an input byte >= nsyms                  */
  float ms;                  /* device time of the call (CUDA events)                    */
} fsm_batch_result;

uint64_t fsm_batch_chunks(const uint64_t* h_offsets, uint32_t nstreams, uint32_t chunk_bytes);
int fsm_run_batch(fsm_t fsm, const uint8_t* d_input, const uint64_t* h_offsets, uint32_t nstreams,
                  const fsm_run_opts* opts, uint32_t* d_final, uint64_t* d_count, uint32_t* d_chunk_ends,
                  fsm_batch_result* out);

/* Paper-literal SRE (Alg. 2 L2-6 + Alg. 3, P:98-102, P:162-179,
 * verbatim): ONE CTA, one thread per chunk, a shared `mark`, one frontier step per
 * iteration with a CTA barrier, exactly N iterations; a must-do recovery is one
 * thread's walk of its chunk.  A reference point for fsm_run's batched-frontier
 * design (same results; R13).  Only opts->chunk_bytes, vr_end and stream
 * are used (VR_tid = one FIFO list of vr_end records).  d_input / d_chunk_ends as in
 * fsm_run.  Synchronous.  Errors: FSM_EUNSUPPORTED when ceil(len / chunk_bytes) >
 * 1024; FSM_ESYMBOL as fsm_run.  Stats: rounds = iterations with a must-do recovery,
 * tasks_* = re-executions, verify_* over all N iterations, ms_verify = kernel time. */
int fsm_run_literal(fsm_t fsm, const uint8_t* d_input, uint64_t len, const fsm_run_opts* opts,
                    uint32_t* d_chunk_ends, fsm_result* out);

/* FSM-level batching (Alg. 1 L2-3): npairs (DFA, stream)
 * pairs — fsms[i] over d_inputs[i][0, lens[i]) (device pointers, any alignment) — in ONE
 * launch per table format: one CTA per pair stages that DFA's table in shared memory and
 * runs lookback-2 speculation + SRE rounds over the pair's stream in waves of 256 chunks
 * (opts->chunk_bytes; other opts ignored).  Handles may repeat.  Writes h_final[i]
 * (original id; 0xFFFFFFFF when the stream holds a symbol >= nsyms, and the call then
 * returns FSM_ESYMBOL after filling every output) and h_count[i] (accept count).  out
 * (nullable): re-walks, SRE rounds, kernel milliseconds.  Synchronous on opts->stream. */
typedef struct {
  uint64_t rewalks;  /* chunk re-executions over all pairs          */
  uint64_t rounds;   /* SRE rounds with a re-execution, summed       */
  float ms;          /* device time of the launches (CUDA events)    */
} fsm_multi_result;
int fsm_run_multi(const fsm_t* fsms, uint32_t npairs, const uint8_t* const* d_inputs, const uint64_t* lens,
                  const fsm_run_opts* opts, uint32_t* h_final, uint64_t* h_count, fsm_multi_result* out);

/* Same as fsm_run with HOST buffers: copies h_input to the device (pinned
 * memory recommended), runs, and copies chunk ends back to h_chunk_ends
 * (nullable).  Used for end-to-end timing. */
int fsm_run_host(fsm_t fsm, const uint8_t* h_input, uint64_t len, const fsm_run_opts* opts,
                 uint32_t* h_chunk_ends, fsm_result* out);

/* Scheme selector: profile the device sample (the paper uses a
 * 1 MB trace), compute the features, walk the decision tree (Fig. 6,
 * reconstructed: DESIGN.md R19) and cache the choice for FSM_SCHEME_AUTO.
 * A sample longer than 1 MiB (e.g. the whole stream) is profiled on 8 portions
 * of 128 KiB spread evenly over it — portion i at floor(i (len - 128 KiB) / 7)
 * rounded down to 4 KiB — gathered into one 1 MiB sample (reading R20: input
 * sensitivity compares "different portions").  FSM_SCHEME_AUTO without a
 * cached choice profiles the run's own input this way.  feat nullable. */
int fsm_select_scheme(fsm_t fsm, const uint8_t* d_sample, uint64_t len, const fsm_run_opts* opts,
                      fsm_scheme* out, fsm_features* feat);

/* The chunk-size rule of reading R29 for a stream of stream_len bytes per GPU, from the
 * convergence fractions of features filled by fsm_select_scheme (e.g. when the profile
 * was a sample of a longer stream): the smallest W in {4096, 8192, 16384} with
 * conv{W} >= 3/4 and stream_len / W >= SMs x 768 (W = 4096 exempt), else 4096.
 * Host-only; the current device's SM count.  NULL -> 4096. */
uint32_t fsm_chunk_for(const fsm_features* feat, uint64_t stream_len);

/* ---- multi-GPU contiguous sharding --------------------
 * A shard is a contiguous, chunk-aligned byte range [offset, offset+len) of
 * the global stream.  Each rank reduces its shard to a state map over all
 * nstates+1 transformed states (poison included), exchanges the maps with
 * one allgather (NCCL via the caller's process group), composes them, and
 * fixes its chunk ends.  Map layout (device, caller-allocated, fsm_map_bytes()
 * bytes): uint32 end[nt] (0xFFFFFFFF = start not reachable/not computed),
 * then uint64 count[nt].  The poison state (nt-1, R4) is a fixed entry of every
 * map (poison -> poison, count 0), so an invalid byte in any shard makes every
 * rank's fsm_shard_finish return FSM_ESYMBOL, as fsm_run does.  */
uint64_t fsm_map_bytes(fsm_t fsm);
/* Step 1 (per rank): d_shard = shard bytes; d_lookback = the up to 2 bytes
 * before the shard (NULL/0 for the first shard, whose start is q0).  Writes
 * the map to d_map; chunk ends that do not depend on the shard's start state
 * go to d_chunk_ends_local (device, nullable, fsm_num_chunks(len) entries),
 * the rest is kept in the handle for fsm_shard_finish.  On failure the call
 * returns its status AND writes an error map (every entry 0xFFFFFFFD, count[0] =
 * -status) when d_map is valid: the caller must still take part in the exchange
 * and call fsm_shard_finish, which then returns that status on every rank — no
 * rank is left waiting in the collective.  Non-convergent DFAs above the ENUM
 * limit (paths that never merge) run one pipeline per surviving path: exact, at
 * (#paths) x the shard's work. */
int fsm_shard_map(fsm_t fsm, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback,
                  uint32_t lookback_len, const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local);
/* fsm_shard_map is speculative for a shard with a lookback: its pipeline is queued
 * from the first candidate without waiting to learn whether every candidate's path
 * merged with it (P:427 path fusion) — no host round trip.  If one did not, the map
 * is marked invalid and fsm_shard_finish returns FSM_EAGAIN on EVERY rank; every rank
 * then calls fsm_shard_map_exact (same arguments: checks on the host, falls back to
 * per-path pipelines or enumeration), exchanges the maps again and finishes. */
int fsm_shard_map_exact(fsm_t fsm, const uint8_t* d_shard, uint64_t len, const uint8_t* d_lookback,
                        uint32_t lookback_len, const fsm_run_opts* opts, void* d_map, uint32_t* d_chunk_ends_local);
/* Step 2 (every rank, after the allgather): d_maps = nranks maps back to back.
 * Composes them from q0 (s_{g+1} = M_g[s_g]), writes this rank's chunk ends
 * (original ids, nullable) and the global result.  FSM_EAGAIN: see above.
 * A failed map on any rank: that rank's status on every rank. */
int fsm_shard_finish(fsm_t fsm, const void* d_maps, uint32_t nranks, uint32_t rank,
                     const fsm_run_opts* opts, uint32_t* d_chunk_ends_local, fsm_result* out_global);

/* Asynchronous step 2: queues the composition and the fix-up on opts->stream and
 * returns a ticket at once (the host fix-up modes of non-merging shards finish here and
 * the ticket carries the outcome); fsm_shard_wait blocks until that step is done and
 * fills *out.  Steps on one handle may be queued back to back (up to 32 in flight), so
 * the host never stalls the GPU between steps.  FSM_EAGAIN from the wait: redo the step
 * synchronously (fsm_run_sharded / fsm_shard_map_exact) on every rank. */
int fsm_shard_finish_async(fsm_t fsm, const void* d_maps, uint32_t nranks, uint32_t rank,
                           const fsm_run_opts* opts, uint32_t* d_chunk_ends_local, uint64_t* ticket);
int fsm_shard_wait(fsm_t fsm, uint64_t ticket, fsm_result* out);

/* ---- library-owned NCCL path (callers without torch.distributed) -------------
 * fsm_comm_unique_id (one rank, 128 bytes, share out of band) -> fsm_comm_init
 * on every rank (one GPU each) -> fsm_run_sharded = fsm_shard_map + one
 * ncclAllGather of the maps on opts->stream + fsm_shard_finish.  NCCL is
 * loaded at run time (libnccl.so.2); FSM_ENCCL if it is missing or fails. */
typedef struct fsm_comm_s* fsm_comm_t;
int fsm_comm_unique_id(void* id_out);
/* device: the CUDA device of this rank (cudaSetDevice), -1 = the current one. */
int fsm_comm_init(int nranks, int rank, const void* unique_id, int device, fsm_comm_t* out);
int fsm_run_sharded(fsm_t fsm, fsm_comm_t comm, const uint8_t* d_shard, uint64_t shard_len,
                    const uint8_t* d_lookback, uint32_t lookback_len, const fsm_run_opts* opts,
                    uint32_t* d_chunk_ends_local, fsm_result* out_global);
/* fsm_run_sharded without the host wait: map + ncclAllGather + fsm_shard_finish_async;
 * collect with fsm_shard_wait(fsm, ticket, out). */
int fsm_run_sharded_async(fsm_t fsm, fsm_comm_t comm, const uint8_t* d_shard, uint64_t shard_len,
                          const uint8_t* d_lookback, uint32_t lookback_len, const fsm_run_opts* opts,
                          uint32_t* d_chunk_ends_local, uint64_t* ticket);
/* The SURVEY §8(b) form: the shard's offset and the stream's length instead of lookback
 * bytes — the library gathers every rank's last 16 bytes (one tiny ncclAllGather, a host
 * wait) and takes the 16 bytes before this shard from the nearest preceding non-empty
 * shards.  shard_offset must be a multiple of chunk_bytes.  Then as fsm_run_sharded. */
int fsm_run_sharded_at(fsm_t fsm, fsm_comm_t comm, const uint8_t* d_shard, uint64_t shard_offset,
                       uint64_t shard_len, uint64_t total_len, const fsm_run_opts* opts,
                       uint32_t* d_chunk_ends_local, fsm_result* out_global);
void fsm_comm_free(fsm_comm_t comm);

/* ---- peer-memory exchange (no collective library) ---------------
 * The fused alternative of SURVEY §8(e): each rank owns a mailbox in its HBM (two
 * step-parity sets of nranks map slots + arrival flags) that every peer maps through
 * CUDA IPC (peer memory over NVLink / NVSwitch).  fsm_p2p_create allocates it and
 * returns its 64-byte IPC handle; the caller exchanges the handles out of band (e.g.
 * torch.distributed all_gather_object) and passes all nranks of them, in rank order, to
 * fsm_p2p_open.  fsm_run_sharded_p2p = fsm_shard_map into the own slot, one kernel that
 * stores the map into every peer's mailbox and raises its flag there, one kernel that
 * waits (bounded: FSM_ENCCL after ~10 s) for every peer's flag, then fsm_shard_finish
 * over the own mailbox.  Same results and error protocol as fsm_run_sharded.  One
 * fsm_p2p_t per (handle, rank); every rank must run the same sequence of steps. */
typedef struct fsm_p2p_s* fsm_p2p_t;
int fsm_p2p_create(fsm_t fsm, int nranks, int rank, void* ipc_handle_out, fsm_p2p_t* out);
int fsm_p2p_open(fsm_p2p_t p2p, const void* ipc_handles);
int fsm_run_sharded_p2p(fsm_t fsm, fsm_p2p_t p2p, const uint8_t* d_shard, uint64_t shard_len,
                        const uint8_t* d_lookback, uint32_t lookback_len, const fsm_run_opts* opts,
                        uint32_t* d_chunk_ends_local, fsm_result* out_global);
void fsm_p2p_free(fsm_p2p_t p2p);

/* ---- introspection (tests) ------------------------------------------------- */
/* perm/inv: host uint32 [nstates+1] (poison = nstates last); freq: uint64
 * [nstates]; mode/H/C: table format, hot rows, classes. Any pointer nullable. */
int fsm_get_transform(fsm_t fsm, uint32_t* perm, uint32_t* inv, uint64_t* freq, uint32_t* mode,
                      uint32_t* hot_rows, uint32_t* nclasses);
/* Ranked lookback candidates QS (transformed ids) for the symbol pair (a, b). */
int fsm_get_qs(fsm_t fsm, uint8_t a, uint8_t b, uint32_t* qs, uint32_t* qs_len, uint32_t* image_size);

/* Records of the last fsm_run (hierarchical store, level 3), for tests: host
 * arrays of [32 slots][nchunks] (slot s < 16: VR^end ring, s >= 16: VR^others
 * ring) in TRANSFORMED ids, plus per-chunk ring counts and x[0..nchunks]
 * (incoming states).  Any pointer nullable. */
int fsm_get_records(fsm_t fsm, uint64_t nchunks, uint32_t* start, uint32_t* end, uint32_t* cnt, uint32_t* n_end,
                    uint32_t* n_oth, uint32_t* x);

/* Phase timeline of the last collected run's verify/recover kernel (profiling):
 * us[i] = microseconds since kernel start at phase boundary i (stage table,
 * each relaxation pass, each recovery, finalize); up to 24 entries. */
int fsm_get_phase_times(fsm_t fsm, double* us, uint32_t* n);

/* Run timeline of the last collected run (profiling; recorded only when the
 * environment has GSPEC_STAMPS=1 at library load, otherwise every entry is -1):
 * us[0] = speculative-execution kernel (entry of CTA 0 -> last warp done),
 * us[1] = gap until the verify/recover kernel's entry, us[2] = verify/recover
 * kernel (entry -> last CTA done).  us: caller-owned, 3 doubles. */
int fsm_get_timeline(fsm_t fsm, double* us);

void fsm_free(fsm_t fsm);
const char* fsm_strerror(int status);
const char* fsm_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
