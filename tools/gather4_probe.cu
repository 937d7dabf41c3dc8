// gather4_probe.cu — does TMA tile::gather4 (4 arbitrary rows x 64 B, box {64, 1})
// with SWIZZLE_64B land rows in shared memory with the same address-based XOR
// pattern as a 32-row 2-D box (the layout k_spec_tma's readers assume), at
// 256-byte destination offsets?  And what input rate does a warp-per-32-rows
// gather4 pipeline reach over a 1 GiB [N][4096] stream with scattered rows?
// nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/g4 tools/gather4_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void g4(uint32_t dst, const CUtensorMap* tm, uint32_t bar, int x, int r0, int r1, int r2,
                                   int r3) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, "
      "%5, %6}], [%7];" ::"r"(dst),
      "l"(tm), "r"(x), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void wait(uint32_t bar, uint32_t ph) {
  uint32_t done = 0;
  while (!done)
    asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0,1,0,p;\n}\n"
                 : "=r"(done)
                 : "r"(bar), "r"(ph)
                 : "memory");
}

__global__ void k_layout(const __grid_constant__ CUtensorMap tm, uint8_t* out, int off) {
  __shared__ __align__(1024) uint8_t buf[2048];
  __shared__ uint64_t bar;
  for (int i = threadIdx.x; i < 2048; i++) buf[i] = 0xEE;
  if (threadIdx.x == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)));
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&bar)), "r"(256));
    g4(sa(buf + off), &tm, sa(&bar), 128, 5, 100, 7, 900);
  }
  wait(sa(&bar), 0);
  __syncthreads();
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) out[i] = buf[i];
}

// each warp: stages of 32 rows (8 gather4 ops by lane 0), rows = a scattered permutation
template <int S>
__global__ void __launch_bounds__(512, 1) k_rate(const __grid_constant__ CUtensorMap tm, const uint32_t* rows,
                                                 uint32_t nrows, uint32_t segs, unsigned long long* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const uint32_t w = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  uint8_t* st = sm + w * S * 2048;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + nw * S * 2048) + w * S;
  if (lane == 0)
    for (int s = 0; s < S; s++) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(bars + s)));
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  const uint32_t gw = blockIdx.x * nw + w, tw = gridDim.x * nw;
  const uint32_t ngroups = nrows / 32;
  uint32_t acc = 0;
  uint64_t items = 0;
  for (uint32_t g = gw; g < ngroups; g += tw) items += segs;
  uint32_t pg = gw, psg = 0, ps = 0;
  auto issue = [&]() {
    const uint32_t* r = rows + pg * 32;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(bars + ps)), "r"(2048));
    for (int q = 0; q < 8; q++)
      g4(sa(st + ps * 2048 + q * 256), &tm, sa(bars + ps), psg * 64, r[4 * q], r[4 * q + 1], r[4 * q + 2],
         r[4 * q + 3]);
    if (++psg == segs) { psg = 0; pg += tw; }
    if (++ps == S) ps = 0;
  };
  if (lane == 0)
    for (uint64_t i = 0; i < items && i < S; i++) issue();
  uint32_t s = 0, ph = 0;
  for (uint64_t i = 0; i < items; i++) {
    wait(sa(bars + s), ph);
    const uint4 v = *reinterpret_cast<const uint4*>(st + s * 2048 + lane * 64);
    acc += v.x ^ v.y ^ v.z ^ v.w;
    __syncwarp();
    if (lane == 0 && i + S < items) issue();
    if (++s == S) { s = 0; ph ^= 1; }
  }
  if (acc == 0x12345678u) sink[0] = acc;
}

int main() {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = reinterpret_cast<CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                           const cuuint64_t*, const cuuint32_t*, const cuuint32_t*,
                                           CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                           CUtensorMapFloatOOBfill)>(fn);
  const uint64_t B = 4096, N = (1ull << 30) / B;
  uint8_t* d;
  cudaMalloc(&d, N * B);
  std::vector<uint8_t> h(1024 * B);
  for (size_t i = 0; i < h.size(); i++) h[i] = (uint8_t)((i / B) * 7 + (i % B) / 16);  // row r, 16B unit u
  cudaMemcpy(d, h.data(), h.size(), cudaMemcpyHostToDevice);
  for (int sw = 0; sw < 2; sw++) {
    CUtensorMap tm;
    cuuint64_t dims[2] = {B, N}, str[1] = {B};
    cuuint32_t box[2] = {64, 1}, es[2] = {1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     sw ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("swizzle=%d encode=%d\n", sw, (int)r);
    uint8_t* o;
    cudaMalloc(&o, 2048);
    for (int off : {0, 256, 512, 768}) {
      k_layout<<<1, 128>>>(tm, o, off);
      cudaError_t e = cudaDeviceSynchronize();
      std::vector<uint8_t> hb(2048);
      cudaMemcpy(hb.data(), o, 2048, cudaMemcpyDeviceToHost);
      // expected: row k (0..3) of the op at byte (off + k*64 + (u ^ ((addr>>7)&3))*16) under address-based SWIZZLE_64B
      const int rws[4] = {5, 100, 7, 900};
      int bad_abs = 0, bad_plain = 0;
      for (int k = 0; k < 4; k++)
        for (int u = 0; u < 4; u++) {
          const uint8_t want = (uint8_t)(rws[k] * 7 + (128 / 16) + u);
          const int a = off + k * 64;
          const int pos_abs = a + ((u ^ ((a >> 7) & 3)) * 16);
          const int pos_plain = a + u * 16;
          for (int b = 0; b < 16; b++) {
            bad_abs += hb[pos_abs + b] != want;
            bad_plain += hb[pos_plain + b] != want;
          }
        }
      printf("  off=%d err=%s  mismatches: address-swizzled %d, plain %d\n", off, cudaGetErrorString(e), bad_abs,
             bad_plain);
    }
    if (!sw) continue;
    // rate: scattered permutation of rows, 32 rows per warp-stage
    std::vector<uint32_t> perm(N);
    for (uint64_t i = 0; i < N; i++) perm[i] = (uint32_t)i;
    srand(1);
    for (uint64_t i = N - 1; i > 0; i--) std::swap(perm[i], perm[rand() % (i + 1)]);
    for (int sparse : {0, 1}) {
      uint32_t nr = sparse ? (uint32_t)(N * 4 / 10) : (uint32_t)N;
      nr &= ~31u;
      uint32_t* dr;
      cudaMalloc(&dr, nr * 4);
      cudaMemcpy(dr, perm.data(), nr * 4, cudaMemcpyHostToDevice);
      unsigned long long* sink;
      cudaMalloc(&sink, 8);
      for (int warps : {16, 24}) {
        const int S = 3;
        const size_t smem = warps * S * 2048 + warps * S * 8;
        cudaFuncSetAttribute(k_rate<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        float best = 1e9;
        for (int it = 0; it < 5; it++) {
          cudaEventRecord(a);
          k_rate<3><<<148, warps * 32, smem>>>(tm, dr, nr, (uint32_t)(B / 64), sink);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          float t;
          cudaEventElapsedTime(&t, a, b);
          if (t < best) best = t;
        }
        printf("rate rows=%u (%s) warps=%d: %.3f ms, %.0f GB/s (%s)\n", nr, sparse ? "40%" : "all", warps, best,
               (double)nr * B / best / 1e6, cudaGetErrorString(cudaGetLastError()));
      }
      cudaFree(dr);
    }
  }
  return 0;
}
