// gen_cuda.cu — device twin of gs_input_fill (gen.c): same bytes, generated in
// HBM so multi-GiB bench inputs need no host->device copy.  Test/bench
// infrastructure only; the product library never links this.
#include <cuda_runtime.h>

#include "gen.h"
#include "gs_hash.h"

namespace {

__constant__ uint8_t c_skew[2][256];

__global__ void k_background(uint32_t kind, uint32_t nsyms, uint64_t seed, uint32_t sensitive,
                             uint64_t offset, uint64_t len, uint8_t* __restrict__ out) {
  // one thread per aligned 8-byte group of the absolute stream
  uint64_t g0 = offset >> 3, g1 = (offset + len + 7) >> 3;
  for (uint64_t g = g0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < g1;
       g += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t h = (kind == GS_IN_UNIFORM) ? gs_hash(seed ^ GS_SALT_RAND, g) : gs_hash(seed, g);
    for (int k = 0; k < 8; k++) {
      uint64_t i = g * 8 + k;
      if (i < offset || i >= offset + len) continue;
      uint8_t v;
      if (kind == GS_IN_BITS) {
        v = (uint8_t)((gs_hash(seed, i >> 6) >> (i & 63)) & 1);
      } else if (kind == GS_IN_UNIFORM) {
        v = (uint8_t)(((h >> (8 * k)) & 0xff) % nsyms);
      } else {
        int var = (sensitive && ((i >> GS_REGION_LOG2) & 1)) ? 1 : 0;
        v = c_skew[var][(h >> (8 * k)) & 0xff];
      }
      out[i - offset] = v;
    }
  }
}

__global__ void k_plants(uint64_t seed, uint32_t ppb, uint32_t nlit, const uint8_t* __restrict__ lb,
                         const uint32_t* __restrict__ lo, uint64_t offset, uint64_t len,
                         uint8_t* __restrict__ out) {
  const uint64_t bs = 1ULL << GS_PLANT_BLOCK_LOG2;
  uint64_t end = offset + len;
  uint64_t b0 = offset >> GS_PLANT_BLOCK_LOG2, b1 = (end - 1) >> GS_PLANT_BLOCK_LOG2;
  for (uint64_t b = b0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; b <= b1;
       b += (uint64_t)gridDim.x * blockDim.x) {
    for (uint32_t j = 0; j < ppb; j++) {  // sequential per block: later plants win
      uint64_t h = gs_hash(seed ^ GS_SALT_PLANT, b * ppb + j);
      uint32_t l = (uint32_t)(h % nlit);
      uint32_t ll = lo[l + 1] - lo[l];
      uint64_t pos = b * bs + (uint64_t)((h >> 32) % (bs - ll + 1));
      for (uint32_t t = 0; t < ll; t++) {
        uint64_t q = pos + t;
        if (q >= offset && q < end) out[q - offset] = lb[lo[l] + t];
      }
    }
  }
}

__global__ void k_resets(uint64_t seed, int32_t rb, uint64_t offset, uint64_t len, uint8_t* __restrict__ out) {
  uint64_t end = offset + len;
  uint64_t r0 = offset >> GS_RESET_BLOCK_LOG2, r1 = (end - 1) >> GS_RESET_BLOCK_LOG2;
  for (uint64_t r = r0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r <= r1;
       r += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t q = (r << GS_RESET_BLOCK_LOG2) +
                 (gs_hash(seed ^ GS_SALT_RESET, r) & ((1ULL << GS_RESET_BLOCK_LOG2) - 1));
    if (q >= offset && q < end) out[q - offset] = (uint8_t)rb;
  }
}

}  // namespace

extern "C" int gs_input_fill_device(const gs_input_params* p, uint64_t offset, uint64_t len,
                                    uint8_t* d_out, void* stream) {
  if (len == 0) return 0;
  cudaStream_t st = (cudaStream_t)stream;
  uint8_t skew[2][256];
  gs_skew_table(0, skew[0]);
  gs_skew_table(1, skew[1]);
  if (cudaMemcpyToSymbolAsync(c_skew, skew, sizeof(skew), 0, cudaMemcpyHostToDevice, st) != cudaSuccess)
    return -3;
  uint32_t ns = p->nsyms ? p->nsyms : 256;
  k_background<<<148 * 8, 256, 0, st>>>(p->kind, ns, p->seed, p->sensitive, offset, len, d_out);
  if (p->kind == GS_IN_TEXT && p->plants_per_block && p->nlit) {
    uint32_t tot = p->lit_off[p->nlit];
    uint8_t* dlb = nullptr;
    uint32_t* dlo = nullptr;
    if (cudaMallocAsync((void**)&dlb, tot + 1, st) != cudaSuccess) return -2;
    if (cudaMallocAsync((void**)&dlo, sizeof(uint32_t) * (p->nlit + 1), st) != cudaSuccess) return -2;
    cudaMemcpyAsync(dlb, p->lit_bytes, tot, cudaMemcpyHostToDevice, st);
    cudaMemcpyAsync(dlo, p->lit_off, sizeof(uint32_t) * (p->nlit + 1), cudaMemcpyHostToDevice, st);
    k_plants<<<148 * 4, 256, 0, st>>>(p->seed, p->plants_per_block, p->nlit, dlb, dlo, offset, len, d_out);
    cudaFreeAsync(dlb, st);
    cudaFreeAsync(dlo, st);
  }
  if (p->kind == GS_IN_TEXT && p->reset_byte >= 0)
    k_resets<<<148 * 2, 256, 0, st>>>(p->seed, p->reset_byte, offset, len, d_out);
  // the host copies above read caller memory: finish before returning
  if (cudaStreamSynchronize(st) != cudaSuccess) return -3;
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
