// Probe: gap between two dependent kernels on one stream — the second launched normally vs
// cooperatively (grid = SMs x 2 CTAs of 256 threads), the first a long-running full-GPU kernel.
// Prints the %globaltimer gap between the last CTA of kernel A and the first CTA of kernel B.
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;
__device__ unsigned long long g_end_a, g_start_b;
__device__ __forceinline__ unsigned long long gt() { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__global__ void kA(int iters) {
  float x = threadIdx.x;
  for (int i = 0; i < iters; i++) x = x * 1.0001f + 0.5f;
  if (x == 12345.f) printf("x");
  __syncthreads();
  if (threadIdx.x == 0) atomicMax(&g_end_a, gt());
}
__global__ void kB_normal() { if (threadIdx.x == 0) atomicMin(&g_start_b, gt()); }
__global__ void kB_coop() { if (threadIdx.x == 0) atomicMin(&g_start_b, gt()); cg::this_grid().sync(); }
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaStream_t st; cudaStreamCreate(&st);
  for (int mode = 0; mode < 2; mode++) {
    double sum = 0; int n = 0;
    for (int r = 0; r < 30; r++) {
      unsigned long long z = 0, m = ~0ull;
      cudaMemcpyToSymbol(g_end_a, &z, 8); cudaMemcpyToSymbol(g_start_b, &m, 8);
      kA<<<sms, 1024, 0, st>>>(20000);
      if (mode == 0) kB_normal<<<sms * 2, 256, 0, st>>>();
      else { void* args[] = {nullptr}; cudaLaunchCooperativeKernel((void*)kB_coop, sms * 2, 256, args, 0, st); }
      cudaStreamSynchronize(st);
      unsigned long long a, b; cudaMemcpyFromSymbol(&a, g_end_a, 8); cudaMemcpyFromSymbol(&b, g_start_b, 8);
      if (r >= 5) { sum += (double)(b - a); n++; }
    }
    printf("%s launch: mean gap %.2f us\n", mode ? "cooperative" : "normal", sum / n / 1000.0);
  }
  return 0;
}
