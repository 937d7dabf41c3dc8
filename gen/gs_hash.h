/* gs_hash.h — counter-based hash shared by the host generator (gen.c) and its
 * CUDA twin (gen_cuda.cu).  This module holds NO part of the method's
 * arithmetic (no DFA walks, no speculation): it only turns (seed, counter)
 * into pseudo-random bits, so host and device produce byte-identical inputs.
 *
 * splitmix64 finaliser (Steele, Lea, Flood 2014) applied to seed + (ctr+1)*phi.
 */
#ifndef GS_HASH_H
#define GS_HASH_H
#include <stdint.h>

#if defined(__CUDACC__)
#define GS_HD __host__ __device__ __forceinline__
#else
#define GS_HD static inline
#endif

GS_HD uint64_t gs_mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

GS_HD uint64_t gs_hash(uint64_t seed, uint64_t ctr) {
  return gs_mix64(seed + (ctr + 1ULL) * 0x9E3779B97F4A7C15ULL);
}

/* salts separating the independent random streams of one input recipe */
#define GS_SALT_PLANT 0x504C414E54ULL  /* "PLANT" */
#define GS_SALT_RESET 0x5245534554ULL  /* "RESET" */
#define GS_SALT_LIT 0x4C4954ULL        /* "LIT"   */
#define GS_SALT_RAND 0x52414E44ULL     /* "RAND"  */

#define GS_PLANT_BLOCK_LOG2 12 /* plants are decided per 4 KiB block     */
#define GS_RESET_BLOCK_LOG2 13 /* one reset byte per 8 KiB block        */
#define GS_REGION_LOG2 26      /* input-sensitive regions of 64 MiB     */

#endif
