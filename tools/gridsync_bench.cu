// Grid barrier cost on B200: cooperative_groups grid.sync() vs a hand-rolled
// sense-reversing barrier (one atomic per CTA + spin on a generation word).
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;

__global__ void k_cg(int iters, int* sink) {
  cg::grid_group g = cg::this_grid();
  for (int i = 0; i < iters; i++) g.sync();
  if (threadIdx.x == 0 && blockIdx.x == 0) *sink = iters;
}

__device__ __forceinline__ void my_sync(unsigned* bar, unsigned nb, unsigned& gen) {
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned g0 = gen;
    __threadfence();
    unsigned a = atomicAdd(bar, 1);
    if (a == nb - 1) {
      atomicExch(bar, 0);
      __threadfence();
      atomicExch(bar + 1, g0 + 1);
    } else {
      while (*(volatile unsigned*)(bar + 1) == g0) {}
    }
    __threadfence();
  }
  gen++;
  __syncthreads();
}

__global__ void k_my(int iters, unsigned* bar, int* sink) {
  unsigned gen = *(volatile unsigned*)(bar + 1);
  for (int i = 0; i < iters; i++) my_sync(bar, gridDim.x, gen);
  if (threadIdx.x == 0 && blockIdx.x == 0) *sink = iters;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int* sink;
  unsigned* bar;
  cudaMalloc(&sink, 4);
  cudaMalloc(&bar, 8);
  cudaMemset(bar, 0, 8);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int per : {1, 2, 4}) {
    for (int thr : {256, 512, 1024}) {
      if (per * thr > 2048) continue;
      int grid = sms * per, iters = 2000;
      void* args[] = {&iters, &sink};
      cudaLaunchCooperativeKernel((void*)k_cg, grid, thr, args, 0, 0);
      cudaEventRecord(a);
      cudaLaunchCooperativeKernel((void*)k_cg, grid, thr, args, 0, 0);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      void* args2[] = {&iters, &bar, &sink};
      cudaLaunchCooperativeKernel((void*)k_my, grid, thr, args2, 0, 0);
      cudaEventRecord(a);
      cudaLaunchCooperativeKernel((void*)k_my, grid, thr, args2, 0, 0);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms2;
      cudaEventElapsedTime(&ms2, a, b);
      printf("grid %4d x %4d: cg %.3f us/sync, custom %.3f us/sync (%s)\n", grid, thr, 1e3 * ms / iters,
             1e3 * ms2 / iters, cudaGetErrorString(cudaGetLastError()));
    }
  }
  // empty cooperative launch latency
  int iters = 0;
  void* args[] = {&iters, &sink};
  cudaEventRecord(a);
  for (int i = 0; i < 100; i++) cudaLaunchCooperativeKernel((void*)k_cg, sms, 512, args, 0, 0);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  printf("empty cooperative launch (back to back): %.2f us\n", 1e3 * ms / 100);
  return 0;
}
