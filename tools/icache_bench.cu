// Cold-code cost on B200: one warp runs N instructions of straight-line code
// (a fully unrolled dependent integer chain) right after a 256 MiB L2 flush
// ("cold": the code comes from HBM) or right after running the same kernel
// ("warm").  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
// tools/icache_bench.cu -o tools/icache_bench
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
template <int N>
__global__ void straight(unsigned* io, unsigned long long* t, int nblk) {
  if (blockIdx.x >= nblk) return;
  unsigned x = io[threadIdx.x];
  const unsigned long long t0 = gt();
#pragma unroll
  for (int i = 0; i < N; i++) x = x * 1664525u + (unsigned)i;
  const unsigned long long t1 = gt();
  io[threadIdx.x + 32] = x;
  if (threadIdx.x == 0) t[blockIdx.x] = t1 - t0;
}
__global__ void flush(uint4* b, size_t n) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = make_uint4(i, 0, 0, 0);
}
template <int N>
void run(unsigned* io, unsigned long long* t, uint4* fb) {
  for (int nblk : {1, 148}) {
    for (int cold = 1; cold >= 0; cold--) {
      unsigned long long best = ~0ull, h[148];
      for (int rep = 0; rep < 5; rep++) {
        if (cold) flush<<<1184, 512>>>(fb, (256u << 20) / 16);
        else straight<N><<<148, 32>>>(io, t, nblk);
        cudaDeviceSynchronize();
        straight<N><<<148, 32>>>(io, t, nblk);
        cudaDeviceSynchronize();
        cudaMemcpy(h, t, nblk * 8, cudaMemcpyDeviceToHost);
        unsigned long long mx = 0;
        for (int b = 0; b < nblk; b++) mx = mx > h[b] ? mx : h[b];
        best = best < mx ? best : mx;
      }
      printf("N=%6d straight-line steps (~%3d KB of SASS)  CTAs %3d  %s  %8.2f us  (%.1f ns per KB)\n", N,
             N * 2 * 16 / 1024, nblk, cold ? "cold (L2 flushed)" : "warm             ", best / 1e3,
             best / (N * 2 * 16 / 1024.0));
    }
  }
}
int main() {
  unsigned* io;
  unsigned long long* t;
  uint4* fb;
  cudaMalloc(&io, 4096);
  cudaMemset(io, 1, 4096);
  cudaMalloc(&t, 148 * 8);
  cudaMalloc(&fb, 256u << 20);
  run<1024>(io, t, fb);
  run<4096>(io, t, fb);
  run<16384>(io, t, fb);
  return 0;
}
