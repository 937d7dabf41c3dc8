/* oracle.h — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, sequential CPU implementation of what GSpecPal's hot path
 * computes (PAPER.md = /root/reference/PAPER.md; "P:n" = line n there).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  It shares no code, header, table or
 * constant with the CUDA path (paper_conf_ipps_wangwqw22_b200/csrc) and never
 * calls it.  Pins: tests/test_oracle_*.py.
 *
 * Conventions: DFA tables are row-major uint32 [n][nsyms] in ORIGINAL state
 * ids unless a function says "transformed".  Status codes mirror gspec.h's
 * values but are defined independently here.
 */
#ifndef GS_ORACLE_H
#define GS_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define OR_OK 0
#define OR_EINVAL (-1)
#define OR_ESYMBOL (-4)
#define OR_EUNSUPPORTED (-6)

/* Alg. 1 FSM_PROCESSING on a DFA, recording the state after
 * the last symbol of every chunk of B bytes (reading c.4 #2) and counting the
 * positions whose state is accepting (reading c.4 #3). chunk_end may be NULL. */
int or_run(const uint32_t* table, uint32_t n, uint32_t nsyms, uint32_t q0, const uint8_t* accept,
           const uint8_t* in, uint64_t len, uint32_t B, uint32_t* chunk_end,
           uint32_t* final_state, uint64_t* accept_count);

/* Frequency-based DFA transformation (Fig. 4).
 * policy 0: freq = static in-degree in the table; policy 1: visit counts of a
 * sequential walk over `profile` (north_star "visit frequency").  Ranks by
 * (-freq, original id); perm[q] = rank, inv[rank] = q.  The poison state
 * (index n, absorbing, reached by symbols >= nsyms) is ranked last: perm has
 * n+1 entries, inv n+1.  tt (transformed table, [n+1][nsyms]) and acc_t
 * ([n+1]) may be NULL.  freq may be NULL. */
int or_transform(const uint32_t* table, uint32_t n, uint32_t nsyms, const uint8_t* accept, int policy,
                 const uint8_t* profile, uint64_t profile_len, uint32_t q0,
                 uint32_t* perm, uint32_t* inv, uint64_t* freq, uint32_t* tt, uint8_t* acc_t);

/* All-state lookback (§IV-A): run every state q < nq of the table
 * `t` (any numbering; nq = number of real states, poison excluded) over w[0..L);
 * rank the distinct results by (-multiplicity, id), keep the first K in qs.
 * Returns the number of distinct results (image size).  If any symbol of w is
 * >= nsyms the image is {poison} with poison = nq. */
uint32_t or_lookback(const uint32_t* t, uint32_t nq, uint32_t nsyms, const uint8_t* w, uint32_t L,
                     uint32_t K, uint32_t* qs, uint32_t* qs_len);

/* Lookback of L in [2, 16] symbols (P:300 with L > 2; reading R25): or_lookback over the
 * L symbols w[0..L) before a chunk, except that when the image of the first two of them
 * already has more than 64 states the lookback-2 ranking of the last two (w[L-2..L)) is
 * used — the cost bound of the GPU path; both images contain the true start. */
uint32_t or_lookback_long(const uint32_t* t, uint32_t nq, uint32_t nsyms, const uint8_t* w, uint32_t L,
                          uint32_t K, uint32_t* qs, uint32_t* qs_len);

/* Enumeration: M[q] = state after the chunk from q, C[q] = accepts
 * along that path, for every q < n.  Returns OR_ESYMBOL on an invalid byte. */
int or_enum(const uint32_t* table, uint32_t n, uint32_t nsyms, const uint8_t* accept,
            const uint8_t* in, uint64_t len, uint32_t* M, uint64_t* C);

/* (M2,C2) o (M1,C1): first chunk 1 then chunk 2. */
void or_compose(uint32_t n, const uint32_t* M1, const uint64_t* C1, const uint32_t* M2, const uint64_t* C2,
                uint32_t* M, uint64_t* C);

/* Scheme ids (mirror of the C ABI's enum, restated). */
#define OR_SEQ 1
#define OR_PM 2
#define OR_SRE 3
#define OR_RR 4
#define OR_NF 5
#define OR_ENUM 6
/* Convergence-set enumeration (the exact-coverage methods the
 * paper cites beside SRE, P:427 [21][24]): round 0 runs EVERY lookback candidate
 * of QS_c up to spec_k (the whole lookback image when it has <= spec_k states,
 * which contains the true start), then SRE rounds for whatever a capped
 * image missed. */
#define OR_CSE 7

typedef struct {
  uint32_t final_state; /* original id */
  uint32_t accept;
  uint64_t accept_count;
  uint64_t nchunks;
  uint32_t rounds;
  uint64_t tasks_total, tasks_mustdo, tasks_sre, tasks_helper;
  uint64_t reread_bytes, verify_checks, verify_matches;
  uint64_t active_sum; /* sum over rounds of active workers */
} or_sim_result;

/* One task of the deterministic round semantics. */
typedef struct {
  uint32_t round, chunk, start, kind; /* kind 0 must-do, 1 SRE, 2 helper; start transformed */
} or_task;

/* Deterministic round semantics of Alg. 2-5 (SURVEY c.3)
 * on the TRANSFORMED DFA (tt, acc_t, q0t, nt = real states, poison = nt).
 * scheme: OR_SEQ/PM/SRE/RR/NF.  chunk_end (nullable) gets ORIGINAL ids via inv.
 * tasks (nullable) receives up to max_tasks task records. */
int or_simulate(const uint32_t* tt, uint32_t nt, uint32_t nsyms, uint32_t q0t, const uint8_t* acc_t,
                const uint32_t* inv, const uint8_t* in, uint64_t len, uint32_t B, int scheme,
                uint32_t spec_k, uint32_t qs_cap, uint32_t lookback, uint32_t vr_end, uint32_t vr_oth,
                uint32_t* chunk_end, or_sim_result* res, or_task* tasks, uint64_t max_tasks,
                uint64_t* ntasks);

/* Paper-literal SRE (Alg. 2 L2-6 + Alg. 3 verbatim, one frontier step per iteration,
 * exactly N iterations).  Same outputs as or_run; diagnostics: rounds =
 * iterations with a must-do recovery, tasks_total = re-executions. */
int or_simulate_literal_sre(const uint32_t* tt, uint32_t nt, uint32_t nsyms, uint32_t q0t, const uint8_t* acc_t,
                            const uint32_t* inv, const uint8_t* in, uint64_t len, uint32_t B, uint32_t vr_cap,
                            uint32_t* chunk_end, or_sim_result* res);

/* Paper-literal RR (Alg. 4) and NF (Alg. 5) — and SRE (Alg. 3)
 * through the same loop: N iterations of Alg. 3's frontier step, the recovery step of
 * the chosen algorithm when mark == false.  Per-iteration task log (nullable):
 * tasks[i] = {iteration, chunk, start, kind 0 must-do / 1 rear / 2 helper}. */
int or_simulate_literal(const uint32_t* tt, uint32_t nt, uint32_t nsyms, uint32_t q0t, const uint8_t* acc_t,
                        const uint32_t* inv, const uint8_t* in, uint64_t len, uint32_t B, int scheme,
                        uint32_t qs_cap, uint32_t vr_cap, uint32_t* chunk_end, or_sim_result* res, or_task* tasks,
                        uint64_t max_tasks, uint64_t* ntasks);

/* Faithful PM (Parallel Merge, Xia et al., the paper's prior state of the art; P:120-127,
 * Fig. 2, Eq. 2).  spec-k round 0; stage 1: log N rounds of a
 * parallel tree-like verification and merge of the chunks' k-entry maps, a mismatch
 * marking the path invalid (delayed recovery, no re-execution); stage 2: sequential
 * verification from q0 over the merged segments, with an immediate recovery of a chunk
 * whose incoming state has no (valid) record.  Same outputs as or_run. */
typedef struct {
  uint32_t levels;          /* tree rounds = ceil(log2 N) */
  uint64_t merge_checks;    /* left entries looked up among a right segment's starts */
  uint64_t invalid_marks;   /* entries marked invalid by a merge (delayed recovery) */
  uint64_t jumps;           /* stage 2: segments taken through their merged map */
  uint64_t recoveries;      /* stage 2: must-be-done re-executions (P_i^PM events) */
  uint64_t reread_bytes;
} or_pm_stats;

int or_simulate_pm_tree(const uint32_t* tt, uint32_t nt, uint32_t nsyms, uint32_t q0t, const uint8_t* acc_t,
                        const uint32_t* inv, const uint8_t* in, uint64_t len, uint32_t B, uint32_t k,
                        uint32_t qs_cap, uint32_t* chunk_end, or_sim_result* res, or_pm_stats* pm);

typedef struct {
  double acc1, acck, sens, uniq10;
} or_features;

/* Selector features (reading c.4 #19) on the TRANSFORMED DFA. */
int or_features_compute(const uint32_t* tt, uint32_t nt, uint32_t nsyms, uint32_t q0t, const uint8_t* acc_t,
                        const uint8_t* in, uint64_t len, uint32_t B, uint32_t k, uint32_t qs_cap,
                        or_features* out);

/* Convergence lengths of the lookback image over 4 KiB-spaced windows (reading
 * R29).  Returns the number of windows; d_out nullable. */
uint32_t or_conv_lengths(const uint32_t* tt, uint32_t nt, uint32_t nsyms, const uint8_t* in, uint64_t len,
                         uint32_t wmax, uint32_t* d_out);

/* Chunk size from the convergence lengths (reading R29). */
uint32_t or_select_chunk(const uint32_t* d, uint32_t nwin, uint64_t len, uint64_t min_chunks);

/* Decision tree (Fig. 6 reconstructed, reading c.4 #19). Returns a scheme id. */
int or_select(const or_features* f, uint32_t nstates);
/* variant 0 = or_select; 1 = the reconstructed tree without the B200 gate R19b. */
int or_select_variant(const or_features* f, uint32_t nstates, int variant);

#ifdef __cplusplus
}
#endif
#endif
