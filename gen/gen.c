/* gen.c — host side of the seeded workload generators (see gen.h). */
#include "gen.h"

#include <stdlib.h>
#include <string.h>

#include "gs_hash.h"

static const char kLitAlphabet[] = "abcdefghijklmnopqrstuvwxyz0123456789./:_-";

void gs_skew_table(int variant, uint8_t out[256]) {
  /* 256 slots: space 38, '\n' 4, letters 150 (English-like), digits 20,
   * punctuation 22, upper-case 22.  Variant 1 maps vowels to the next letter. */
  static const struct { char c; int w; } letters[26] = {
      {'e', 19}, {'t', 14}, {'a', 12}, {'o', 11}, {'i', 10}, {'n', 10}, {'s', 9},
      {'h', 9},  {'r', 9},  {'d', 6},  {'l', 6},  {'c', 4},  {'u', 4},  {'m', 4},
      {'w', 3},  {'f', 3},  {'g', 3},  {'y', 3},  {'p', 3},  {'b', 2},  {'v', 1},
      {'k', 1},  {'j', 1},  {'x', 1},  {'q', 1},  {'z', 1}};
  static const struct { char c; int w; } punct[6] = {
      {'.', 6}, {'/', 4}, {':', 3}, {'_', 2}, {'-', 3}, {',', 4}};
  int k = 0, i, j;
  for (i = 0; i < 38; i++) out[k++] = ' ';
  for (i = 0; i < 4; i++) out[k++] = '\n';
  for (i = 0; i < 26; i++)
    for (j = 0; j < letters[i].w; j++) {
      char c = letters[i].c;
      if (variant == 1 && (c == 'a' || c == 'e' || c == 'i' || c == 'o' || c == 'u')) c = (char)(c + 1);
      out[k++] = (uint8_t)c;
    }
  for (i = 0; i < 10; i++) { out[k++] = (uint8_t)('0' + i); out[k++] = (uint8_t)('0' + i); }
  for (i = 0; i < 6; i++)
    for (j = 0; j < punct[i].w; j++) out[k++] = (uint8_t)punct[i].c;
  for (i = 0; k < 256; i++) out[k++] = (uint8_t)('A' + i);
}

uint32_t gs_literals(uint64_t seed, uint32_t nlit, uint32_t lmin, uint32_t lmax,
                     uint8_t* out_bytes, uint32_t* out_off) {
  uint32_t pos = 0, i, j;
  if (lmax > 63) lmax = 63;
  if (lmin > lmax) lmin = lmax;
  for (i = 0; i < nlit; i++) {
    uint64_t h = gs_hash(seed ^ GS_SALT_LIT, (uint64_t)i * 64);
    uint32_t len = lmin + (uint32_t)(h % (uint64_t)(lmax - lmin + 1));
    out_off[i] = pos;
    for (j = 0; j < len; j++)
      out_bytes[pos++] = (uint8_t)kLitAlphabet[gs_hash(seed ^ GS_SALT_LIT, (uint64_t)i * 64 + 1 + j) % 41];
  }
  out_off[nlit] = pos;
  return pos;
}

uint64_t gs_bytes_hash(const uint8_t* b, uint64_t len) {
  uint64_t h = 0xcbf29ce484222325ULL, i;
  for (i = 0; i < len; i++) { h ^= b[i]; h *= 0x100000001b3ULL; }
  return h;
}

void gs_input_fill(const gs_input_params* p, uint64_t offset, uint64_t len, uint8_t* out) {
  uint64_t i, end = offset + len;
  if (len == 0) return;
  if (p->kind == GS_IN_BITS) {
    for (i = offset; i < end; i++) out[i - offset] = (uint8_t)((gs_hash(p->seed, i >> 6) >> (i & 63)) & 1);
    return;
  }
  if (p->kind == GS_IN_UNIFORM) {
    uint32_t ns = p->nsyms ? p->nsyms : 256;
    for (i = offset; i < end; i++)
      out[i - offset] = (uint8_t)(((gs_hash(p->seed ^ GS_SALT_RAND, i >> 3) >> (8 * (i & 7))) & 0xff) % ns);
    return;
  }
  /* GS_IN_TEXT: background */
  uint8_t skew[2][256];
  gs_skew_table(0, skew[0]);
  gs_skew_table(1, skew[1]);
  for (i = offset; i < end; i++) {
    int var = (p->sensitive && ((i >> GS_REGION_LOG2) & 1)) ? 1 : 0;
    out[i - offset] = skew[var][(gs_hash(p->seed, i >> 3) >> (8 * (i & 7))) & 0xff];
  }
  /* plants: per 4 KiB block, later plants overwrite earlier ones */
  if (p->plants_per_block && p->nlit) {
    const uint64_t bs = 1ULL << GS_PLANT_BLOCK_LOG2;
    uint64_t b0 = offset >> GS_PLANT_BLOCK_LOG2, b1 = (end - 1) >> GS_PLANT_BLOCK_LOG2, b;
    for (b = b0; b <= b1; b++) {
      uint32_t j;
      for (j = 0; j < p->plants_per_block; j++) {
        uint64_t h = gs_hash(p->seed ^ GS_SALT_PLANT, b * p->plants_per_block + j);
        uint32_t l = (uint32_t)(h % p->nlit);
        uint32_t ll = p->lit_off[l + 1] - p->lit_off[l];
        uint64_t pos = b * bs + (uint64_t)((h >> 32) % (bs - ll + 1));
        uint32_t t;
        for (t = 0; t < ll; t++) {
          uint64_t q = pos + t;
          if (q >= offset && q < end) out[q - offset] = p->lit_bytes[p->lit_off[l] + t];
        }
      }
    }
  }
  /* resets: one per 8 KiB block, after plants */
  if (p->reset_byte >= 0) {
    uint64_t r0 = offset >> GS_RESET_BLOCK_LOG2, r1 = (end - 1) >> GS_RESET_BLOCK_LOG2, r;
    for (r = r0; r <= r1; r++) {
      uint64_t q = (r << GS_RESET_BLOCK_LOG2) + (gs_hash(p->seed ^ GS_SALT_RESET, r) & ((1ULL << GS_RESET_BLOCK_LOG2) - 1));
      if (q >= offset && q < end) out[q - offset] = (uint8_t)p->reset_byte;
    }
  }
}

void gs_dfa_div7(uint32_t table[14], uint8_t accept[7]) {
  /* div7 (Fig. 1): remainder of the binary number read MSB first */
  uint32_t s, b;
  for (s = 0; s < 7; s++) {
    for (b = 0; b < 2; b++) table[s * 2 + b] = (2 * s + b) % 7;
    accept[s] = (s == 0);
  }
}

uint32_t gs_dfa_ac(uint32_t nlit, const uint8_t* lit_bytes, const uint32_t* lit_off,
                   uint32_t* table, uint8_t* accept) {
  /* Aho & Corasick 1975: trie + failure links; delta(u,c) = goto(u,c) or delta(fail(u),c) */
  uint32_t maxn = 1 + lit_off[nlit], n = 1, i, t, c;
  int32_t* go = (int32_t*)malloc(sizeof(int32_t) * 256 * (size_t)maxn);
  uint8_t* out = (uint8_t*)calloc(maxn, 1);
  uint32_t* fail = (uint32_t*)calloc(maxn, sizeof(uint32_t));
  uint32_t* q = (uint32_t*)malloc(sizeof(uint32_t) * maxn);
  uint32_t* d = (uint32_t*)malloc(sizeof(uint32_t) * 256 * (size_t)maxn);
  memset(go, 0xff, sizeof(int32_t) * 256 * (size_t)maxn);
  for (i = 0; i < nlit; i++) {
    uint32_t u = 0;
    for (t = lit_off[i]; t < lit_off[i + 1]; t++) {
      c = lit_bytes[t];
      if (go[u * 256 + c] < 0) go[u * 256 + c] = (int32_t)(n++);
      u = (uint32_t)go[u * 256 + c];
    }
    if (lit_off[i + 1] > lit_off[i]) out[u] = 1;
  }
  if (table) {
    uint32_t qh = 0, qt = 0;
    for (c = 0; c < 256; c++) {
      int32_t v = go[c];
      if (v >= 0) { fail[v] = 0; q[qt++] = (uint32_t)v; d[c] = (uint32_t)v; }
      else d[c] = 0;
    }
    while (qh < qt) {
      uint32_t u = q[qh++];
      out[u] |= out[fail[u]];
      for (c = 0; c < 256; c++) {
        int32_t v = go[u * 256 + c];
        if (v >= 0) {
          fail[v] = d[fail[u] * 256 + c];
          d[u * 256 + c] = (uint32_t)v;
          q[qt++] = (uint32_t)v;
        } else {
          d[u * 256 + c] = d[fail[u] * 256 + c];
        }
      }
    }
    memcpy(table, d, sizeof(uint32_t) * 256 * (size_t)n);
    memcpy(accept, out, n);
  }
  free(go); free(out); free(fail); free(q); free(d);
  return n;
}

static int is_vowel(uint32_t c) { return c == 'a' || c == 'e' || c == 'i' || c == 'o' || c == 'u'; }

uint32_t gs_dfa_ac_counter(uint32_t nlit, const uint8_t* lit_bytes, const uint32_t* lit_off,
                           int32_t reset_byte, uint32_t* table, uint8_t* accept) {
  uint32_t na = gs_dfa_ac(nlit, lit_bytes, lit_off, NULL, NULL), a, k, c;
  if (!table) return na * 16;
  uint32_t* ta = (uint32_t*)malloc(sizeof(uint32_t) * 256 * (size_t)na);
  uint8_t* fa = (uint8_t*)malloc(na);
  gs_dfa_ac(nlit, lit_bytes, lit_off, ta, fa);
  for (a = 0; a < na; a++)
    for (k = 0; k < 16; k++) {
      uint32_t s = a * 16 + k;
      for (c = 0; c < 256; c++) {
        uint32_t k2 = ((int32_t)c == reset_byte) ? 0 : (is_vowel(c) ? (k + 1) & 15 : k);
        table[(size_t)s * 256 + c] = ta[(size_t)a * 256 + c] * 16 + k2;
      }
      accept[s] = (uint8_t)(fa[a] && k == 0);
    }
  free(ta); free(fa);
  return na * 16;
}

void gs_dfa_random(uint64_t seed, uint32_t n, uint32_t nsyms, uint32_t* table, uint8_t* accept) {
  uint64_t i;
  for (i = 0; i < (uint64_t)n * nsyms; i++) table[i] = (uint32_t)(gs_hash(seed ^ GS_SALT_RAND, i) % n);
  for (i = 0; i < n; i++) accept[i] = (uint8_t)(gs_hash(seed ^ GS_SALT_RAND ^ 1, i) & 1);
}
