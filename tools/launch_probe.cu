// launch_probe.cu — per-launch overhead of plain vs cooperative launches (B200).
// nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/lp tools/launch_probe.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__global__ void k_empty(int* p) { if (p && threadIdx.x == 0 && blockIdx.x == 0) p[0] = 1; }
__global__ void k_sync(int* p, int n) {
  auto g = cg::this_grid();
  for (int i = 0; i < n; i++) g.sync();
  if (p && threadIdx.x == 0 && blockIdx.x == 0) p[0] = 1;
}

int main() {
  int* d; cudaMalloc(&d, 4);
  cudaStream_t s; cudaStreamCreate(&s);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int reps = 200;
  for (int bps : {1, 2, 5}) {
    for (int bs : {256, 896}) {
      if (bs == 896 && bps > 1) continue;
      const int grid = sms * bps;
      float t;
      for (int w = 0; w < 2; w++) {
        cudaEventRecord(a, s);
        for (int i = 0; i < reps; i++) k_empty<<<grid, bs, 0, s>>>(d);
        cudaEventRecord(b, s); cudaEventSynchronize(b); cudaEventElapsedTime(&t, a, b);
      }
      printf("grid %4d x %3d plain empty        %.2f us/launch\n", grid, bs, 1000 * t / reps);
      for (int ns : {0, 1, 4}) {
        void* args[] = {&d, (void*)&ns};
        for (int w = 0; w < 2; w++) {
          cudaEventRecord(a, s);
          for (int i = 0; i < reps; i++) cudaLaunchCooperativeKernel((void*)k_sync, grid, bs, args, 0, s);
          cudaEventRecord(b, s); cudaEventSynchronize(b); cudaEventElapsedTime(&t, a, b);
        }
        printf("grid %4d x %3d cooperative %d syncs %.2f us/launch (%s)\n", grid, bs, ns, 1000 * t / reps,
               cudaGetErrorString(cudaGetLastError()));
      }
    }
  }
  return 0;
}
