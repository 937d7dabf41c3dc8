// spec_exec.cu — B2: partition + lookback speculation + parallel speculative
// execution (Alg. 2 L2-6; spec-k for PM).
//
// Each thread owns NI consecutive chunks and walks KP paths per chunk, so a
// thread keeps NI*KP independent transition chains in flight (ILP).  Chunk
// c >= 1 starts from QS_c[0..k) read from the lookback-2 pair table;
// chunk 0 starts at q0.  The transformed table sits in shared memory
// (P:317-330).  Output: round-0 records (VR^end) and x[c+1] = the
// speculative end of chunk c.
#include <cstdlib>
#include <string>

#include "internal.h"
#include "walk.cuh"

namespace gspec {

bool spec_path_generic_only() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("GSPEC_SPEC_PATH");
    v = (e && std::string(e) == "generic") ? 1 : 0;
  }
  return v == 1;
}

namespace {

template <int MODE, int NI, int KP>
__global__ void __launch_bounds__(256) k_spec_exec(DevImage img, RunParams rp, RecStore rs, uint64_t c0) {
  extern __shared__ __align__(1024) uint8_t smem[];
  stage_table(img, smem);
  if (rp.ctl_init && blockIdx.x == 0) init_ctl(rp.ctl_init, q0_of(rp), rp.N);
  __syncthreads();
  using S = Step<MODE>;
  const uint64_t N = rp.N, B = rp.B, len = rp.len;
  const uint64_t ngroups = (N - c0 + NI - 1) / NI;
  const bool aligned = (reinterpret_cast<uintptr_t>(rp.in) & 15u) == 0;
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < ngroups;
       g += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t c[NI];
    uint32_t st[NI][KP], code[NI][KP], acc[NI][KP], kc[NI];
    bool all_full = aligned;
#pragma unroll
    for (int i = 0; i < NI; i++) {
      c[i] = c0 + g * NI + i;
      const bool valid = c[i] < N;
      all_full &= valid && (c[i] + 1) * B <= len;
      if (!valid || c[i] == 0) {
        kc[i] = 1;
#pragma unroll
        for (int p = 0; p < KP; p++) st[i][p] = q0_of(rp);
      } else {
        uint32_t ql;
        const uint32_t* qs = qs_chunk(img, rp, c[i], &ql);
        kc[i] = min(rp.k, min(ql, rp.qs_cap));
#pragma unroll
        for (int p = 0; p < KP; p++) st[i][p] = __ldg(qs + min((uint32_t)p, kc[i] - 1));
      }
#pragma unroll
      for (int p = 0; p < KP; p++) {
        code[i][p] = __ldg(img.tid2code + st[i][p]);
        acc[i][p] = 0;
      }
    }
    if (all_full) {
      const uint4* v[NI];
#pragma unroll
      for (int i = 0; i < NI; i++) v[i] = reinterpret_cast<const uint4*>(rp.in + c[i] * B);
      const uint32_t nv = (uint32_t)(B / 16);
      uint4 q[NI];
#pragma unroll
      for (int i = 0; i < NI; i++) q[i] = __ldg(v[i]);
      for (uint32_t j = 0; j < nv; j++) {
        uint4 cur[NI];
#pragma unroll
        for (int i = 0; i < NI; i++) {
          cur[i] = q[i];
          if (j + 1 < nv) q[i] = __ldg(v[i] + j + 1);  // prefetch the next 16 bytes
        }
#pragma unroll
        for (int t = 0; t < 4; t++) {
          uint32_t w[NI];
#pragma unroll
          for (int i = 0; i < NI; i++) w[i] = t == 0 ? cur[i].x : t == 1 ? cur[i].y : t == 2 ? cur[i].z : cur[i].w;
#pragma unroll
          for (int i = 0; i < NI; i++)
#pragma unroll
            for (int p = 0; p < KP; p++) { code[i][p] = S::template word<0>(img, smem, code[i][p], w[i]); acc[i][p] += S::acc(code[i][p]); }
#pragma unroll
          for (int i = 0; i < NI; i++)
#pragma unroll
            for (int p = 0; p < KP; p++) { code[i][p] = S::template word<1>(img, smem, code[i][p], w[i]); acc[i][p] += S::acc(code[i][p]); }
#pragma unroll
          for (int i = 0; i < NI; i++)
#pragma unroll
            for (int p = 0; p < KP; p++) { code[i][p] = S::template word<2>(img, smem, code[i][p], w[i]); acc[i][p] += S::acc(code[i][p]); }
#pragma unroll
          for (int i = 0; i < NI; i++)
#pragma unroll
            for (int p = 0; p < KP; p++) { code[i][p] = S::template word<3>(img, smem, code[i][p], w[i]); acc[i][p] += S::acc(code[i][p]); }
        }
      }
    } else {
#pragma unroll
      for (int i = 0; i < NI; i++) {
        if (c[i] >= N) continue;
        const uint64_t lo = c[i] * B, n = min(B, len - lo);
#pragma unroll
        for (int p = 0; p < KP; p++) code[i][p] = walk_bytes<MODE>(img, smem, rp.in + lo, n, code[i][p], acc[i][p]);
      }
    }
#pragma unroll
    for (int i = 0; i < NI; i++) {
      if (c[i] >= N) continue;
      const uint64_t cc = c[i];
      uint32_t e0 = 0;
#pragma unroll
      for (int p = 0; p < KP; p++) {
        const uint32_t e = S::tid(img, code[i][p]);
        if (p == 0) e0 = e;
        if ((uint32_t)p < kc[i]) {
          rs.start[p * rs.cap + cc] = st[i][p];
          rs.end[p * rs.cap + cc] = e;
          rs.cnt[p * rs.cap + cc] = acc[i][p];
        }
      }
      rs.n_end[cc] = kc[i];
      rs.n_oth[cc] = 0;
      rs.next_qs[cc] = (uint8_t)kc[i];
      rs.ref_start[cc] = st[i][0];
      rs.ref_end[cc] = e0;
      rs.ref_cnt[cc] = acc[i][0];
      rs.x[cc + 1] = e0;
      rs.cur_end[cc] = e0;
      if (cc == 0) rs.x[0] = q0_of(rp);
    }
  }
}

template <int MODE, int NI, int KP>
cudaError_t launch_t(const DevImage& img, const RunParams& rp, const RecStore& rs, cudaStream_t st, uint64_t c0) {
  auto kern = k_spec_exec<MODE, NI, KP>;
  const uint32_t smem = smem_bytes_for(img);
  int occ = 0;
  const int sms = device_sms();
  cudaError_t e = kernel_setup((const void*)kern, smem, 256, &occ);
  if (e != cudaSuccess) return e;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  const uint64_t groups = (rp.N - c0 + NI - 1) / NI;
  uint64_t want = (groups + 255) / 256;
  uint64_t grid = (uint64_t)sms * occ;
  if (want < grid) grid = want;
  if (grid < 1) grid = 1;
  kern<<<(unsigned)grid, 256, smem, st>>>(img, rp, rs, c0);
  return cudaGetLastError();
}

template <int MODE>
cudaError_t launch_mode(const DevImage& img, const RunParams& rp, const RecStore& rs, cudaStream_t st, uint64_t c0) {
  if (rp.k <= 1) return launch_t<MODE, 2, 1>(img, rp, rs, st, c0);
  if (rp.k <= 2) return launch_t<MODE, 1, 2>(img, rp, rs, st, c0);
  if (rp.k <= 4) return launch_t<MODE, 1, 4>(img, rp, rs, st, c0);
  if (rp.k <= 8) return launch_t<MODE, 1, 8>(img, rp, rs, st, c0);
  return launch_t<MODE, 1, 16>(img, rp, rs, st, c0);
}

}  // namespace

cudaError_t launch_spec_generic(const DevImage& img, const RunParams& rp, const RecStore& rs, cudaStream_t st,
                                uint64_t c0) {
  if (c0 >= rp.N) return cudaSuccess;
  switch (img.mode) {
    case MODE_U8: return launch_mode<MODE_U8>(img, rp, rs, st, c0);
    case MODE_U16: return launch_mode<MODE_U16>(img, rp, rs, st, c0);
    case MODE_U16H: return launch_mode<MODE_U16H>(img, rp, rs, st, c0);
    case MODE_U16D: return launch_mode<MODE_U16D>(img, rp, rs, st, c0);
    default: return launch_mode<MODE_U32>(img, rp, rs, st, c0);
  }
}

cudaError_t launch_spec_exec(const DevImage& img, const RunParams& rp, const RecStore& rs, cudaStream_t st,
                             uint64_t* tma_done) {
  if (tma_done) *tma_done = 0;
  if (rp.N == 0) return cudaSuccess;
  const int sms = device_sms();
  uint64_t done = 0;
  cudaError_t e = spec_path_generic_only() ? cudaErrorNotSupported : launch_spec_tma(img, rp, rs, sms, st, &done);
  if (e != cudaSuccess && e != cudaErrorNotSupported) return e;
  if (tma_done && e == cudaSuccess) *tma_done = done;
  RunParams rp2 = rp;
  if (e == cudaErrorNotSupported) {
    cudaGetLastError();  // clear
    done = 0;
  } else {
    rp2.ctl_init = nullptr;  // already initialised by the TMA kernel
  }
  if (done >= rp.N) return cudaSuccess;
  return launch_spec_generic(img, rp2, rs, st, done);  // tail chunk (or everything)
}

}  // namespace gspec
