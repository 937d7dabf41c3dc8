// walk.cuh — the state-transition step of every kernel ("state =
// Table[state][symbol]"), specialised per table format, plus the shared-memory
// staging of the hot part of the transformed table.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace gspec {

// Copy the hot table prefix (and the class map) into dynamic shared memory.
// Layout: u8 mode: [table]; classed modes: [cls: 256 B][table: smem_table_bytes]
// (the class map first keeps it 256-aligned: its address is one PRMT away).
__device__ __forceinline__ void stage_table(const DevImage& img, uint8_t* smem) {
  if (img.mode == MODE_U16D) {  // one image [hot rows][class map][delta rows]; delta offsets made absolute
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
    if (base + 2 * img.HC1 > 0xFFFFu) __trap();  // fsm_load bounds the hot bytes by 64 KiB - kDeltaBaseMax
    const uint4* from = reinterpret_cast<const uint4*>(img.Dl);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    const uint32_t nv = img.smem_table_bytes / 16, d0 = img.delta_off / 16;
    for (uint32_t i = threadIdx.x; i < nv; i += blockDim.x) {
      uint4 v = __ldg(from + i);
      if (i >= d0) {
        v.x += base << 16;
        v.z += base << 16;
      }
      dst[i] = v;
    }
    return;
  }
  const uint4* src = (img.mode == MODE_U8)                                 ? reinterpret_cast<const uint4*>(img.T8)
                     : (img.mode == MODE_U16 || img.mode == MODE_U16H) ? reinterpret_cast<const uint4*>(img.T16)
                                                                         : reinterpret_cast<const uint4*>(img.T32);
  const uint32_t off = img.mode == MODE_U8 ? 0u : 256u;
  uint4* dst = reinterpret_cast<uint4*>(smem + off);
  const uint32_t nv = img.smem_table_bytes / 16;
  for (uint32_t i = threadIdx.x; i < nv; i += blockDim.x) dst[i] = __ldg(src + i);
  if (img.mode != MODE_U8) {
    const uint4* cs = reinterpret_cast<const uint4*>(img.mode == MODE_U16H ? img.cls2 : img.cls);
    uint4* cd = reinterpret_cast<uint4*>(smem);
    for (uint32_t i = threadIdx.x; i < 16; i += blockDim.x) cd[i] = __ldg(cs + i);
  }
}

__host__ __device__ inline uint32_t smem_bytes_for(const DevImage& img) {
  return img.smem_table_bytes + (img.mode == MODE_U8 || img.mode == MODE_U16D ? 0u : 256u);
}

template <int MODE>
struct Step;

// MODE_U8: code < 256 with the accept flag in bit 7 (acc += code >> 7).  Row
// `code` starts at code * kRow8 bytes; the 4-byte pad rotates consecutive
// rows by one bank, so lanes in different states that read the same byte hit
// different banks (lanes in the same state read one row: broadcast or
// distinct banks).
constexpr uint32_t kRow8 = 260;

__device__ __forceinline__ uint32_t lds_u8(uint32_t saddr) {
  uint32_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(saddr));
  return v;
}

// (byte K of w) + base, for a 256-aligned base < 2^24: one PRMT
template <int K>
__device__ __forceinline__ uint32_t byte_plus(uint32_t w, uint32_t base) {
  uint32_t b;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(b) : "r"(w), "r"(base), "n"(0x7650 | K));
  return b;
}

template <>
struct Step<MODE_U8> {
  static constexpr uint32_t kShift = 7;
  // s (the smem table) must be 256-byte aligned: address = code*260 + (base | byte) = PRMT + IMAD
  template <int K>
  static __device__ __forceinline__ uint32_t word(const DevImage&, const uint8_t* s, uint32_t code, uint32_t w) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return lds_u8(code * kRow8 + byte_plus<K>(w, base));
  }
  static __device__ __forceinline__ uint32_t byte(const DevImage&, const uint8_t* s, uint32_t code, uint32_t b) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return lds_u8(base + code * kRow8 + b);
  }
  static __device__ __forceinline__ uint32_t acc(uint32_t code) { return code >> 7; }
  static __device__ __forceinline__ uint32_t tid(const DevImage& img, uint32_t code) { return __ldg(img.code2tid + code); }
  // split step (walk16): the state-independent part of symbol K of w, then the dependent lookup
  template <int K>
  static __device__ __forceinline__ uint32_t cls(const DevImage&, const uint8_t* s, uint32_t w) {
    return byte_plus<K>(w, static_cast<uint32_t>(__cvta_generic_to_shared(s)));
  }
  static __device__ __forceinline__ uint32_t next(const DevImage&, const uint8_t*, uint32_t code, uint32_t cl) {
    return lds_u8(code * kRow8 + cl);
  }
};

__device__ __forceinline__ uint32_t lds_u16(uint32_t saddr) {
  uint32_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=r"(v) : "r"(saddr));
  return v;
}

__device__ __forceinline__ uint32_t lds_u32(uint32_t saddr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr));
  return v;
}

// MODE_U16 / MODE_U16H / MODE_U32: classed rows (smem: [cls][rows]); tid < H is
// hot (smem), else global/L2.  ALLHOT drops the hot test (every row in smem).
template <typename CodeT, int SHIFT, bool ALLHOT>
struct StepClassed {
  static constexpr uint32_t kShift = SHIFT;
  static constexpr uint32_t kMask = (1u << SHIFT) - 1u;
  static __device__ __forceinline__ uint32_t row(const DevImage& img, uint32_t base, uint32_t code, uint32_t cl) {
    const uint32_t t = code & kMask;
    const uint32_t idx = t * img.C + cl;
    if (ALLHOT || t < img.H)
      return sizeof(CodeT) == 2 ? lds_u16(base + 256 + idx * 2) : lds_u32(base + 256 + idx * 4);
    const CodeT* g = (sizeof(CodeT) == 2) ? reinterpret_cast<const CodeT*>(img.T16) : reinterpret_cast<const CodeT*>(img.T32);
    return __ldg(g + idx);
  }
  static __device__ __forceinline__ uint32_t byte(const DevImage& img, const uint8_t* s, uint32_t code, uint32_t b) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return row(img, base, code, lds_u8(base + b));
  }
  template <int K>
  static __device__ __forceinline__ uint32_t word(const DevImage& img, const uint8_t* s, uint32_t code, uint32_t w) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return row(img, base, code, lds_u8(byte_plus<K>(w, base)));  // class map at the 256-aligned base
  }
  static __device__ __forceinline__ uint32_t acc(uint32_t code) { return code >> SHIFT; }
  static __device__ __forceinline__ uint32_t tid(const DevImage&, uint32_t code) { return code & kMask; }
  template <int K>
  static __device__ __forceinline__ uint32_t cls(const DevImage&, const uint8_t* s, uint32_t w) {
    return lds_u8(byte_plus<K>(w, static_cast<uint32_t>(__cvta_generic_to_shared(s))));
  }
  static __device__ __forceinline__ uint32_t next(const DevImage& img, const uint8_t* s, uint32_t code, uint32_t cl) {
    return row(img, static_cast<uint32_t>(__cvta_generic_to_shared(s)), code, cl);
  }
};

__device__ __forceinline__ uint2 lds_u64(uint32_t saddr) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(saddr));
  return v;
}

// MODE_U16D: pre-multiplied codes.  c = code & 0x7FFF; a hot code is
// its row's entry index (t*C), a cold code c >= HC1 owns the 8-byte delta row
// {x = absolute row byte offset << 16 | e1 << 8 | e0, y = code0 | code1 << 16}.  Every
// lane starts from the hot default x = (base + 2c) << 16 | 0xFFFF (no exceptions); the
// delta-row load is predicated on the cold lanes only (hot lanes generate no
// shared-memory traffic for it), then one row entry is read at (x >> 16) + 2*class
// and the exceptions override by select — two dependent shared-memory loads, no L2
// trip, no divergence, and no multiply by C on the path (the class map holds 2*class).
// With two exceptions this form needs ~10 ALU-pipe and ~3 FMA-pipe instructions per symbol
// (ALU and shared pipes co-bound on C4); the one-exception step below needs ~8, which leaves
// the kernel bound by the shared-memory pipe alone.
// EXC = 1 (img.delta_exc == 1, template mode MODE_U16D1): every delta row has one exception
// (y = its code), so the step drops the second compare and select: ~8 instead of ~10
// ALU-pipe instructions per symbol.  The EXC = 2 reader also reads EXC = 1 images (e1 = 0xFF
// never matches an even 2*class), so kernels off the hot path keep Step<MODE_U16D>.
template <int EXC>
struct StepDeltaT {
  static constexpr uint32_t kShift = 15;
  static __device__ __forceinline__ uint32_t row(const DevImage& img, uint32_t base, uint32_t code, uint32_t cl2) {
    const uint32_t c = code & 0x7FFFu;
    uint32_t dx = c * 0x20000u + ((base << 16) | 0xFFFFu), dy = 0;
    uint32_t da;  // c*8 + const on the FMA pipe (keeps the ALU pipe free)
    asm("mad.lo.u32 %0, %1, 8, %2;" : "=r"(da) : "r"(c), "r"(base + img.delta_off - img.HC1 * 8u));
    asm volatile(
        "{\n .reg .pred p;\n setp.ge.u32 p, %2, %3;\n @p ld.shared.v2.u32 {%0, %1}, [%4];\n}\n"
        : "+r"(dx), "+r"(dy)
        : "r"(c), "r"(img.HC1), "r"(da));
    uint32_t v = lds_u16((dx >> 16) + cl2);
    if constexpr (EXC == 1) {
      v = ((dx ^ cl2) & 0xFFu) == 0 ? dy : v;
    } else {
      const uint32_t x = dx ^ (cl2 * 0x101u);
      v = (x & 0xFFu) == 0 ? (dy & 0xFFFFu) : v;
      v = (x & 0xFF00u) == 0 ? (dy >> 16) : v;
    }
    return v;
  }
  static __device__ __forceinline__ uint32_t byte(const DevImage& img, const uint8_t* s, uint32_t code, uint32_t b) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return row(img, base, code, lds_u8(base + img.cls_off + b));
  }
  template <int K>
  static __device__ __forceinline__ uint32_t word(const DevImage& img, const uint8_t* s, uint32_t code, uint32_t w) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return row(img, base, code, lds_u8(byte_plus<K>(w, base + img.cls_off)));  // class map 256-aligned
  }
  static __device__ __forceinline__ uint32_t acc(uint32_t code) { return code >> 15; }
  static __device__ __forceinline__ uint32_t tid(const DevImage& img, uint32_t code) {
    return __ldg(img.code2tid + (code & 0x7FFFu));
  }
  template <int K>
  static __device__ __forceinline__ uint32_t cls(const DevImage& img, const uint8_t* s, uint32_t w) {
    return lds_u8(byte_plus<K>(w, static_cast<uint32_t>(__cvta_generic_to_shared(s)) + img.cls_off));
  }
  static __device__ __forceinline__ uint32_t next(const DevImage& img, const uint8_t* s, uint32_t code, uint32_t cl) {
    return row(img, static_cast<uint32_t>(__cvta_generic_to_shared(s)), code, cl);
  }
};

template <>
struct Step<MODE_U16> : StepClassed<uint16_t, 15, false> {};
template <>
struct Step<MODE_U16D> : StepDeltaT<2> {};
template <>
struct Step<MODE_U16D1> : StepDeltaT<1> {};
// MODE_U16H: every row in shared memory, pre-multiplied codes (code = 2*t*C | accept: the
// row's byte offset with the accept flag in bit 0) and a doubled class map, so the entry
// address is code - (code & 1) + (base + 256 + 2*class): LOP3 + IADD3 on the dependent chain.
struct StepPM {
  static constexpr uint32_t kShift = 0;
  static __device__ __forceinline__ uint32_t row(uint32_t base, uint32_t code, uint32_t cl2) {
    return lds_u16(code - (code & 1u) + (base + 256 + cl2));
  }
  static __device__ __forceinline__ uint32_t byte(const DevImage&, const uint8_t* s, uint32_t code, uint32_t b) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return row(base, code, lds_u8(base + b));
  }
  template <int K>
  static __device__ __forceinline__ uint32_t word(const DevImage&, const uint8_t* s, uint32_t code, uint32_t w) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(s));
    return row(base, code, lds_u8(byte_plus<K>(w, base)));  // class map at the 256-aligned base
  }
  static __device__ __forceinline__ uint32_t acc(uint32_t code) { return code & 1u; }
  static __device__ __forceinline__ uint32_t tid(const DevImage& img, uint32_t code) {
    return __ldg(img.code2tid + (code >> 1));
  }
  template <int K>
  static __device__ __forceinline__ uint32_t cls(const DevImage&, const uint8_t* s, uint32_t w) {
    return lds_u8(byte_plus<K>(w, static_cast<uint32_t>(__cvta_generic_to_shared(s))));
  }
  static __device__ __forceinline__ uint32_t next(const DevImage&, const uint8_t* s, uint32_t code, uint32_t cl) {
    return row(static_cast<uint32_t>(__cvta_generic_to_shared(s)), code, cl);
  }
};

template <>
struct Step<MODE_U16H> : StepPM {};
template <>
struct Step<MODE_U32> : StepClassed<uint32_t, 31, false> {};

// Split walk: the class lookups of NW words (4 NW symbols) do not depend on
// the state, so they are all issued before the dependent row chain (the lookups are asm
// volatile, which keeps source order): the chain is one shared-memory load per symbol
// instead of two, ~half the latency of a lane's walk when too few warps hide it.
template <int MODE, int NW>
__device__ __forceinline__ void cls_words(const DevImage& img, const uint8_t* s, const uint32_t (&w)[NW],
                                          uint32_t (&cl)[4 * NW]) {
  using S = Step<MODE>;
#pragma unroll
  for (int t = 0; t < NW; t++) {
    cl[4 * t + 0] = S::template cls<0>(img, s, w[t]);
    cl[4 * t + 1] = S::template cls<1>(img, s, w[t]);
    cl[4 * t + 2] = S::template cls<2>(img, s, w[t]);
    cl[4 * t + 3] = S::template cls<3>(img, s, w[t]);
  }
}

// one path over 16 staged symbols
template <int MODE>
__device__ __forceinline__ void walk16(const DevImage& img, const uint8_t* s, const uint4& q, uint32_t& code,
                                       uint32_t& acc) {
  using S = Step<MODE>;
  const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
  for (int t = 0; t < 4; t++) {  // a word's 4 class lookups at a time (register pressure at 72)
    const uint32_t u[1] = {w[t]};
    uint32_t cl[4];
    cls_words<MODE, 1>(img, s, u, cl);
#pragma unroll
    for (int i = 0; i < 4; i++) {
      code = S::next(img, s, code, cl[i]);
      acc += S::acc(code);
    }
  }
}

// Multi-symbol step table for the enumerative walk on small alphabets:
// TK[tid][combo] advances K symbols per lookup — K = 8 one-bit symbols (nsyms <= 2) or K = 4
// two-bit symbols (nsyms <= 4); combo packs the K symbols, the first in the lowest bits.
// Rows are 257 words (kTkRow bytes) so row r starts at bank r: lanes in different states that
// read the same combo hit different banks.  A chain's code is its row's byte offset
// (tid * kTkRow); an entry = next code | (accepting states among the K) << 24.
constexpr uint32_t kTkRow = 257 * 4;
__host__ __device__ inline uint32_t tk_off(const DevImage& img) { return (smem_bytes_for(img) + 15u) & ~15u; }

// combo of 8 one-bit symbols (bytes 0/1) in w0, w1: one multiply per word gathers its 4
// bytes' low bits into bits 24-27 (the other partial products occupy single bits below 24:
// no carries), the second word's land in bits 28-31 and are shifted to 4-7
__device__ __forceinline__ uint32_t tk_pack8(uint32_t w0, uint32_t w1) {
  return ((w0 * 0x01020408u) >> 24) | ((w1 * 0x01020408u) >> 20);
}
// combo of 4 two-bit symbols (bytes < 4): b0 + 4 b1 + 16 b2 + 64 b3 in bits 24-31, same argument
__device__ __forceinline__ uint32_t tk_pack4(uint32_t w) { return (w * 0x01041040u) >> 24; }

// every byte of the vector is a symbol the table covers (< 2 for K = 8, < 4 for K = 4)
__device__ __forceinline__ bool tk_vector_ok(const uint4& q, uint32_t K) {
  return ((q.x | q.y | q.z | q.w) & (K == 8 ? 0xFEFEFEFEu : 0xFCFCFCFCu)) == 0;
}

template <int NE>
__device__ __forceinline__ void tk_lookup(uint32_t tkbase, uint32_t combo, uint32_t (&sc)[NE], uint32_t (&acc)[NE],
                                          int np) {
  const uint32_t cb = tkbase + (combo << 2);
#pragma unroll
  for (int q = 0; q < NE; q++) {
    if (q >= np) break;
    const uint32_t e = lds_u32(cb + sc[q]);
    sc[q] = e & 0xFFFFFFu;
    acc[q] += e >> 24;
  }
}

// all (<= 8) chains over one 16-byte vector of one-bit symbols through the packed maps PK
// (DevImage::pk_off): per 8 symbols ONE 8-byte lookup, then each chain takes byte t of it
// with a PRMT (selector = its tid) — next tid in the low nibble, accepting states above
template <int NE>
__device__ __forceinline__ void pk_vector(uint32_t pkbase, const uint4& q, uint32_t (&t)[NE], uint32_t (&acc)[NE]) {
  const uint2 e0 = lds_u64(pkbase + tk_pack8(q.x, q.y) * 8u);
  const uint2 e1 = lds_u64(pkbase + tk_pack8(q.z, q.w) * 8u);
#pragma unroll
  for (int j = 0; j < NE; j++) {
    uint32_t x;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(x) : "r"(e0.x), "r"(e0.y), "r"(t[j]));
    acc[j] += (x >> 4) & 0xFu;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(x) : "r"(e1.x), "r"(e1.y), "r"(x & 0xFu));
    t[j] = x & 0xFu;
    acc[j] += (x >> 4) & 0xFu;
  }
}

// the first np chains over one 16-byte vector (tk_vector_ok) through TK
template <int NE>
__device__ __forceinline__ void tk_vector(uint32_t tkbase, uint32_t K, const uint4& q, uint32_t (&sc)[NE],
                                          uint32_t (&acc)[NE], int np = NE) {
  if (K == 8) {
    tk_lookup<NE>(tkbase, tk_pack8(q.x, q.y), sc, acc, np);
    tk_lookup<NE>(tkbase, tk_pack8(q.z, q.w), sc, acc, np);
  } else {
    tk_lookup<NE>(tkbase, tk_pack4(q.x), sc, acc, np);
    tk_lookup<NE>(tkbase, tk_pack4(q.y), sc, acc, np);
    tk_lookup<NE>(tkbase, tk_pack4(q.z), sc, acc, np);
    tk_lookup<NE>(tkbase, tk_pack4(q.w), sc, acc, np);
  }
}

// Walk one path over [p, p+n) bytes from `code`; returns end code, adds accepts.
template <int MODE>
__device__ __forceinline__ uint32_t walk_bytes(const DevImage& img, const uint8_t* s, const uint8_t* p, uint64_t n,
                                               uint32_t code, uint32_t& acc) {
  using S = Step<MODE>;
  uint64_t i = 0;
  // unaligned start: walk the head bytes one by one up to the next 16-byte boundary
  const uint64_t head = min(n, (uint64_t)((16u - (reinterpret_cast<uintptr_t>(p) & 15u)) & 15u));
  for (; i < head; i++) {
    code = S::byte(img, s, code, __ldg(p + i));
    acc += S::acc(code);
  }
  p += head;
  n -= head;
  i = 0;
  // vector part (16-byte aligned now)
  {
    const uint4* v = reinterpret_cast<const uint4*>(p);
    const uint64_t nv = n / 16;
    // software pipeline: two 16-byte loads in flight ahead of the dependent chain
    uint4 q0 = nv > 0 ? __ldg(v) : make_uint4(0, 0, 0, 0);
    uint4 q1 = nv > 1 ? __ldg(v + 1) : make_uint4(0, 0, 0, 0);
    for (uint64_t j = 0; j < nv; j++) {
      const uint4 q = q0;
      q0 = q1;
      if (j + 2 < nv) q1 = __ldg(v + j + 2);
      walk16<MODE>(img, s, q, code, acc);
    }
    i = nv * 16;
  }
  for (; i < n; i++) {
    code = S::byte(img, s, code, __ldg(p + i));
    acc += S::acc(code);
  }
  return code;
}

// Two independent walks interleaved (ILP 2) over arbitrarily aligned ranges: heads
// byte by byte, then both 16-byte-aligned bodies in lockstep, then each one's rest.
template <int MODE>
__device__ __forceinline__ void walk2_bytes(const DevImage& img, const uint8_t* s, const uint8_t* p0, uint64_t n0,
                                            uint32_t& c0, uint32_t& a0, const uint8_t* p1, uint64_t n1, uint32_t& c1,
                                            uint32_t& a1) {
  using S = Step<MODE>;
  const uint64_t h0 = min(n0, (uint64_t)((16u - (reinterpret_cast<uintptr_t>(p0) & 15u)) & 15u));
  const uint64_t h1 = min(n1, (uint64_t)((16u - (reinterpret_cast<uintptr_t>(p1) & 15u)) & 15u));
  for (uint64_t i = 0; i < h0; i++) { c0 = S::byte(img, s, c0, __ldg(p0 + i)); a0 += S::acc(c0); }
  for (uint64_t i = 0; i < h1; i++) { c1 = S::byte(img, s, c1, __ldg(p1 + i)); a1 += S::acc(c1); }
  p0 += h0; n0 -= h0;
  p1 += h1; n1 -= h1;
  const uint64_t nb = min(n0, n1) / 16;
  const uint4* v0 = reinterpret_cast<const uint4*>(p0);
  const uint4* v1 = reinterpret_cast<const uint4*>(p1);
  uint4 q0 = nb > 0 ? __ldg(v0) : make_uint4(0, 0, 0, 0), q1 = nb > 0 ? __ldg(v1) : make_uint4(0, 0, 0, 0);
  for (uint64_t j = 0; j < nb; j++) {
    const uint4 x0 = q0, x1 = q1;
    if (j + 1 < nb) { q0 = __ldg(v0 + j + 1); q1 = __ldg(v1 + j + 1); }
    const uint32_t w0[4] = {x0.x, x0.y, x0.z, x0.w}, w1[4] = {x1.x, x1.y, x1.z, x1.w};
#pragma unroll
    for (int t = 0; t < 4; t++) {
      const uint32_t u0[1] = {w0[t]}, u1[1] = {w1[t]};
      uint32_t k0[4], k1[4];
      cls_words<MODE, 1>(img, s, u0, k0);
      cls_words<MODE, 1>(img, s, u1, k1);
#pragma unroll
      for (int i = 0; i < 4; i++) {
        c0 = S::next(img, s, c0, k0[i]); a0 += S::acc(c0);
        c1 = S::next(img, s, c1, k1[i]); a1 += S::acc(c1);
      }
    }
  }
  c0 = walk_bytes<MODE>(img, s, p0 + nb * 16, n0 - nb * 16, c0, a0);
  c1 = walk_bytes<MODE>(img, s, p1 + nb * 16, n1 - nb * 16, c1, a1);
}

// PDL (see internal.h): wait for the preceding grid (a no-op without a
// programmatic dependency), and let the next grid in the stream launch.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// ---- coherent (L2) accessors for data written by other CTAs of a persistent kernel
__device__ __forceinline__ uint32_t ld_cg(const uint32_t* p) { return __ldcg(p); }
__device__ __forceinline__ void st_cg(uint32_t* p, uint32_t v) { __stcg(p, v); }

// Look x up in VR_c (END slots then OTH slots).  Returns true on a match.
// Slot 0 and the ring counts are loaded together (one L2 round trip for the
// common single-record chunk), the rest of the rings only if needed.  The
// prefetch half depends on c only, so a thread can issue it for several
// chunks before resolving any (batched relaxation passes).
struct VrPre {
  uint32_t ne, no, s0, e0, c0;
};

__device__ __forceinline__ VrPre vr_prefetch(const RecStore& rs, uint64_t c, bool want_cnt) {
  VrPre p;
  p.ne = ld_cg(rs.n_end + c);
  p.no = ld_cg(rs.n_oth + c);
  p.s0 = ld_cg(rs.start + c);
  p.e0 = ld_cg(rs.end + c);
  p.c0 = want_cnt ? ld_cg(rs.cnt + c) : 0u;
  return p;
}

__device__ __forceinline__ bool vr_resolve(const VrPre& p, const RecStore& rs, uint32_t vr_end, uint32_t vr_oth,
                                           uint64_t c, uint32_t x, uint32_t* end, uint32_t* cnt) {
  if (p.ne >= 1 && p.s0 == x) {
    *end = p.e0;
    if (cnt) *cnt = p.c0;
    return true;
  }
  const uint32_t ne = min(p.ne, vr_end);
  for (uint32_t s = 1; s < ne; s++) {
    if (ld_cg(rs.start + s * rs.cap + c) == x) {
      *end = ld_cg(rs.end + s * rs.cap + c);
      if (cnt) *cnt = ld_cg(rs.cnt + s * rs.cap + c);
      return true;
    }
  }
  const uint32_t no = min(p.no, vr_oth);
  for (uint32_t s = 0; s < no; s++) {
    const uint64_t o = (uint64_t)(kVrMax + s) * rs.cap + c;
    if (ld_cg(rs.start + o) == x) {
      *end = ld_cg(rs.end + o);
      if (cnt) *cnt = ld_cg(rs.cnt + o);
      return true;
    }
  }
  return false;
}

__device__ __forceinline__ bool vr_lookup(const RecStore& rs, uint32_t vr_end, uint32_t vr_oth, uint64_t c,
                                          uint32_t x, uint32_t* end, uint32_t* cnt) {
  return vr_resolve(vr_prefetch(rs, c, cnt != nullptr), rs, vr_end, vr_oth, c, x, end, cnt);
}

// FSM_Processing over chunk c from `start` with path fusion: walk in lockstep
// with the chunk's round-0 path; once the two states coincide the rest of the
// path is known (DFA determinism), so end/count follow from the reference.
constexpr uint32_t kFuseMax = 256;  // bytes walked in lockstep with the reference path

template <int MODE>
__device__ __forceinline__ void task_walk(const DevImage& img, const uint8_t* smem, const RunParams& rp, const RecStore& rs,
                          uint64_t c, uint32_t start, uint32_t* end_out, uint32_t* cnt_out) {
  using S = Step<MODE>;
  const uint64_t lo = c * rp.B, n = min((uint64_t)rp.B, rp.len - lo);
  const uint8_t* p = rp.in + lo;
  const uint32_t rstart = __ldcg(rs.ref_start + c);
  const uint32_t rend = __ldcg(rs.ref_end + c), rcnt = __ldcg(rs.ref_cnt + c);
  if (rstart == start) { *end_out = rend; *cnt_out = rcnt; return; }
  uint32_t code = __ldg(img.tid2code + start), rcode = __ldg(img.tid2code + rstart);
  uint32_t acc = 0, racc = 0;
  uint64_t i = 0;
  const bool aligned = (reinterpret_cast<uintptr_t>(p) & 15u) == 0;
  if (aligned) {
    const uint64_t nf = min(n, (uint64_t)kFuseMax) / 16;
    const uint4* v = reinterpret_cast<const uint4*>(p);
    uint4 q0 = nf > 0 ? __ldg(v) : make_uint4(0, 0, 0, 0);
    uint4 q1 = nf > 1 ? __ldg(v + 1) : make_uint4(0, 0, 0, 0);
    for (uint64_t j = 0; j < nf; j++) {
      const uint4 q = q0;
      q0 = q1;
      if (j + 2 < nf) q1 = __ldg(v + j + 2);
      const uint32_t w[4] = {q.x, q.y, q.z, q.w};
      uint32_t cl[16];  // both paths read the same symbols: one class lookup each
      cls_words<MODE, 4>(img, smem, w, cl);
#pragma unroll
      for (int t = 0; t < 16; t++) {
        code = S::next(img, smem, code, cl[t]); acc += S::acc(code);
        rcode = S::next(img, smem, rcode, cl[t]); racc += S::acc(rcode);
      }
      if (code == rcode) {  // merged somewhere in these 16 bytes: identical from here on
        *end_out = rend;
        *cnt_out = rcnt - racc + acc;
        return;
      }
    }
    i = nf * 16;
  }
  code = walk_bytes<MODE>(img, smem, p + i, n - i, code, acc);
  *end_out = S::tid(img, code);
  *cnt_out = acc;
}

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Chunk 0's start state (a shard's reference candidate may live on the device).
__device__ __forceinline__ uint32_t q0_of(const RunParams& rp) { return rp.q0_dev ? __ldcg(rp.q0_dev) : rp.q0t; }

// Initialise the verify/recover control block for a run (block 0 of the first kernel).
__device__ __forceinline__ void init_ctl(Ctl* ctl, uint32_t q0t, uint64_t N) {
  uint32_t* w = reinterpret_cast<uint32_t*>(ctl);
  for (uint32_t i = threadIdx.x; i < sizeof(Ctl) / 4; i += blockDim.x) w[i] = 0;
  __syncthreads();
  if (threadIdx.x == 0) {
    ctl->f = 0;
    ctl->tf = q0t;
    ctl->fmin = N;
    ctl->it_fm[0] = N;
  }
}

// Ranked lookback candidates of chunk c >= 1 (lookback-2 pair table).
__device__ __forceinline__ uint32_t qs_pair(const DevImage& img, const uint8_t* in, uint64_t c, uint32_t B) {
  uint64_t e = c * (uint64_t)B;
  uint32_t a = __ldg(in + e - 2), b = __ldg(in + e - 1);
  return (uint32_t)__ldg(img.cls + a) * img.C + __ldg(img.cls + b);
}

// QS_c of chunk c >= 1: the lookback-2 pair table, or — with a longer lookback
// (fsm_run_opts.lookback > 2, reading R25) — the per-run table rp.qsc built by
// k_qs_long.  Returns the ranked candidates; *ql = their number (<= kQsMax).
__device__ __forceinline__ const uint32_t* qs_chunk(const DevImage& img, const RunParams& rp, uint64_t c,
                                                    uint32_t* ql) {
  if (rp.qsc) {
    *ql = __ldg(rp.qsc_len + c);
    return rp.qsc + c * kQsMax;
  }
  const uint32_t pair = qs_pair(img, rp.in, c, rp.B);
  *ql = __ldg(img.qs2_len + pair);
  return img.qs2 + (uint64_t)pair * kQsMax;
}

}  // namespace gspec
