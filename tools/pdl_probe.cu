// pdl_probe.cu — does programmatic dependent launch (PDL) hide the launch gap
// between a full-SM kernel and a cooperative kernel (and back)?  B200 probe.
// nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/pdl tools/pdl_probe.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// "spec": one CTA per SM, big smem, busy for ~us microseconds
__global__ void k_a(int* p, unsigned us, int trigger) {
  extern __shared__ int sm[];
  if (trigger) asm volatile("griddepcontrol.wait;" ::: "memory");  // previous B's writes
  if (trigger) asm volatile("griddepcontrol.launch_dependents;");
  sm[threadIdx.x] = threadIdx.x;
  const unsigned long long t0 = gt();
  while (gt() - t0 < us * 1000ull) {}
  __syncthreads();
  if (threadIdx.x == 0) p[blockIdx.x] = sm[5];
}
// "verify": cooperative, waits for A, one grid barrier
__global__ void k_b(int* p, int pdl) {
  extern __shared__ int sm[];
  sm[threadIdx.x] = threadIdx.x;  // prologue (table staging stand-in)
  if (pdl) asm volatile("griddepcontrol.wait;" ::: "memory");
  if (pdl) asm volatile("griddepcontrol.launch_dependents;");
  auto g = cg::this_grid();
  g.sync();
  if (threadIdx.x == 0 && blockIdx.x == 0) p[1000] = p[0] + sm[3];
}

int main() {
  int* d; cudaMalloc(&d, 1 << 20);
  cudaStream_t s; cudaStreamCreate(&s);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int smemA = 200 * 1024, smemB = 48 * 1024;
  cudaFuncSetAttribute(k_a, cudaFuncAttributeMaxDynamicSharedMemorySize, smemA);
  cudaFuncSetAttribute(k_b, cudaFuncAttributeMaxDynamicSharedMemorySize, smemB);
  const int reps = 100;
  for (unsigned us : {0u, 20u}) {
    for (int pdl = 0; pdl < 2; pdl++) {
      float t = 0;
      for (int w = 0; w < 2; w++) {
        cudaEventRecord(a, s);
        for (int i = 0; i < reps; i++) {
          cudaLaunchConfig_t ca = {};
          ca.gridDim = sms; ca.blockDim = 896; ca.dynamicSmemBytes = smemA; ca.stream = s;
          cudaLaunchAttribute aa[1];
          aa[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
          aa[0].val.programmaticStreamSerializationAllowed = 1;
          ca.attrs = aa; ca.numAttrs = pdl ? 1 : 0;
          cudaLaunchKernelEx(&ca, k_a, d, us, pdl);
          cudaLaunchConfig_t cb = {};
          cb.gridDim = 2 * sms; cb.blockDim = 256; cb.dynamicSmemBytes = smemB; cb.stream = s;
          cudaLaunchAttribute ab[2];
          ab[0].id = cudaLaunchAttributeCooperative; ab[0].val.cooperative = 1;
          ab[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
          ab[1].val.programmaticStreamSerializationAllowed = 1;
          cb.attrs = ab; cb.numAttrs = pdl ? 2 : 1;
          cudaLaunchKernelEx(&cb, k_b, d, pdl);
        }
        cudaEventRecord(b, s); cudaEventSynchronize(b); cudaEventElapsedTime(&t, a, b);
      }
      printf("busy %2u us  pdl %d : %.2f us per A+B pair (%s)\n", us, pdl, 1000 * t / reps,
             cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
