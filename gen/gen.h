/* gen.h — seeded synthetic workload generators (DFAs and input streams).
 *
 * This module serves BOTH the oracle tests and the CUDA path's tests/bench.
 * It holds none of the method's arithmetic: it builds DFA tables from their
 * textbook definitions (div7, Aho–Corasick, a counter product, random) and
 * input byte streams that are pure functions of (seed, offset), so any slice
 * can be regenerated on host or device (gen_cuda.cu) byte-identically.
 *
 * Workload recipe: SURVEY.md §8.0 and DESIGN.md §"Inputs".
 */
#ifndef GS_GEN_H
#define GS_GEN_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum { GS_IN_BITS = 0, GS_IN_TEXT = 1, GS_IN_UNIFORM = 2 };

typedef struct {
  uint32_t kind;             /* GS_IN_*                                       */
  uint32_t nsyms;            /* GS_IN_UNIFORM: bytes are uniform in [0,nsyms) */
  uint64_t seed;
  uint32_t plants_per_block; /* GS_IN_TEXT: literals planted per 4 KiB block  */
  uint32_t nlit;             /* number of plantable literals                  */
  const uint8_t* lit_bytes;  /* concatenated literal bytes                    */
  const uint32_t* lit_off;   /* [nlit+1] offsets into lit_bytes               */
  int32_t reset_byte;        /* GS_IN_TEXT: -1 none, else 1 per 8 KiB block  */
  uint32_t sensitive;        /* GS_IN_TEXT: odd 64 MiB regions drop vowels    */
} gs_input_params;

/* Fill out[0..len) with bytes offset..offset+len of the stream. */
void gs_input_fill(const gs_input_params* p, uint64_t offset, uint64_t len, uint8_t* out);

/* 64-bit FNV-1a style hash of a byte range (cross-checks host vs device bytes). */
uint64_t gs_bytes_hash(const uint8_t* b, uint64_t len);

/* Background skew table used by GS_IN_TEXT (variant 0 normal, 1 vowel-free). */
void gs_skew_table(int variant, uint8_t out[256]);

/* Literals: nlit literals with lengths in [lmin,lmax] over [a-z0-9./:_-].
 * out_bytes must hold nlit*lmax bytes, out_off nlit+1 entries. Returns total bytes. */
uint32_t gs_literals(uint64_t seed, uint32_t nlit, uint32_t lmin, uint32_t lmax,
                     uint8_t* out_bytes, uint32_t* out_off);

/* DFAs: tables are row-major uint32 [nstates][nsyms], accept uint8 [nstates]. */
void gs_dfa_div7(uint32_t table[7 * 2], uint8_t accept[7]); /* start = 0 */

/* Aho–Corasick automaton over 256 byte symbols. Returns nstates (≤ 1 + total
 * literal bytes) — call with table==NULL to get the size first. start = 0. */
uint32_t gs_dfa_ac(uint32_t nlit, const uint8_t* lit_bytes, const uint32_t* lit_off,
                   uint32_t* table, uint8_t* accept);

/* AC × Z16 counter product (config C3). State (a,k) has id a*16+k; vowels
 * advance k, reset_byte sets k=0; accept iff AC accepts and k==0. start = 0. */
uint32_t gs_dfa_ac_counter(uint32_t nlit, const uint8_t* lit_bytes, const uint32_t* lit_off,
                           int32_t reset_byte, uint32_t* table, uint8_t* accept);

/* Uniform random DFA: every entry uniform in [0,n), accept with prob 1/2. */
void gs_dfa_random(uint64_t seed, uint32_t n, uint32_t nsyms, uint32_t* table, uint8_t* accept);

#ifdef __cplusplus
}
#endif
#endif
