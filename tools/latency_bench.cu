// Dependent-load latency on B200: pointer chases over a random cycle in a
// buffer of `mb` MB, one lane per warp, 2368 warps (the refine grid) or 1,
// with the L2 warm, or after a 256 MiB write (bench.py's L2 flush).  Explains
// the per-phase times of the step (a phase = a few dependent trips).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/latency_bench.cu -o tools/latency_bench
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__global__ void chase(const uint32_t* __restrict__ nxt, int steps, int nw, unsigned long long* out) {
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if ((threadIdx.x & 31) || w >= nw) return;
  uint32_t p = (uint32_t)w * 2654435761u % 1000003u;
  const unsigned long long t0 = gt();
  for (int i = 0; i < steps; i++) p = __ldcg(nxt + p);
  const unsigned long long t1 = gt();
  out[w] = (t1 - t0) | ((unsigned long long)(p & 1) << 63);
}
__global__ void flush(uint8_t* b, size_t n) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n / 16; i += (size_t)gridDim.x * blockDim.x)
    reinterpret_cast<uint4*>(b)[i] = make_uint4(i, 0, 0, 0);
}
int main() {
  uint8_t* fb;
  cudaMalloc(&fb, 256u << 20);
  unsigned long long* out;
  cudaMalloc(&out, 4096 * 8);
  for (size_t mb : {8, 64, 512, 2048}) {
    const size_t n = mb * (1u << 20) / 4;
    std::vector<uint32_t> perm(n), nx(n);
    for (size_t i = 0; i < n; i++) perm[i] = (uint32_t)i;
    std::mt19937 rng(7);
    std::shuffle(perm.begin(), perm.end(), rng);
    for (size_t i = 0; i < n; i++) nx[perm[i]] = perm[(i + 1) % n];
    uint32_t* d;
    cudaMalloc(&d, n * 4);
    cudaMemcpy(d, nx.data(), n * 4, cudaMemcpyHostToDevice);
    for (int nw : {1, 2368})
      for (int fl : {0, 1}) {
        const int steps = 8;
        double sum = 0;
        std::vector<double> v;
        for (int rep = 0; rep < 5; rep++) {
          if (fl) flush<<<1184, 512>>>(fb, 256u << 20);
          else chase<<<148, 512>>>(d, steps, nw, out);  // warm: previous chase touched the lines
          cudaDeviceSynchronize();
          chase<<<148, 512>>>(d, steps, nw, out);
          cudaDeviceSynchronize();
          std::vector<unsigned long long> h(nw);
          cudaMemcpy(h.data(), out, nw * 8, cudaMemcpyDeviceToHost);
          for (auto x : h) v.push_back((x & ~(1ull << 63)) / 1e3 / steps);
        }
        std::sort(v.begin(), v.end());
        printf("buffer %5zu MB  warps %4d  %-12s  per dependent load: median %.2f us  p90 %.2f us\n", mb, nw,
               fl ? "L2 flushed" : "warm", v[v.size() / 2], v[v.size() * 9 / 10]);
      }
    cudaFree(d);
  }
  return 0;
}
