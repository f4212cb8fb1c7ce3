// Same-address / same-line / spread atomics from lane 0 of every warp of a
// 148 x 16-warp grid (the refine kernel's layout): how long the last warp
// waits for its returning atomicAdd.  Build: nvcc -gencode
// arch=compute_100a,code=sm_100a -O3 tools/atomic_bench.cu -o /tmp/atomic_bench
#include <cstdio>
#include <vector>
#include <algorithm>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// mode 0: one address; 1: 8 addresses in one 128-B line (by warp % 8);
// 2: 8 addresses in 8 lines; 3: every warp its own line (no contention)
__global__ void k(int* ctr, unsigned long long* t, int mode, int nact, int ops) {
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if ((threadIdx.x & 31) || w >= nact) return;
  int* p = ctr;
  if (mode == 1) p = ctr + (w & 7);
  if (mode == 2) p = ctr + 32 * (w & 7);
  if (mode == 3) p = ctr + 32 * w;
  const unsigned long long t0 = gt();
  int s = 0;
  for (int i = 0; i < ops; i++) s += atomicAdd(p, 1);
  __threadfence_block();
  if (s < 0) t[1] = 1;  // depend on the returned value before reading the timer
  const unsigned long long t1 = gt();
  t[2 * w] = t0;
  t[2 * w + 1] = t1;
  if (s == -12345) t[0] = 0;  // the returned values are used: a real round trip, not a RED
}

int main() {
  int* ctr;
  unsigned long long* t;
  const int G = 148, T = 512, W = G * T / 32;
  cudaMalloc(&ctr, 32 * W * 4 + 4096);
  cudaMalloc(&t, 2 * W * 8);
  std::vector<unsigned long long> h(2 * W);
  const char* names[] = {"one address", "one line, 8 addresses", "8 lines", "own line per warp"};
  for (int nact : {600, 1100, 2368})
    for (int ops : {1, 2})
      for (int mode = 0; mode < 4; mode++) {
        for (int rep = 0; rep < 3; rep++) {
          cudaMemset(ctr, 0, 32 * W * 4 + 4096);
          cudaMemset(t, 0, 2 * W * 8);
          k<<<G, T>>>(ctr, t, mode, nact, ops);
          cudaDeviceSynchronize();
        }
        cudaMemcpy(h.data(), t, 2 * W * 8, cudaMemcpyDeviceToHost);
        unsigned long long mn = ~0ull, mx = 0;
        std::vector<double> lat;
        for (int w = 0; w < nact; w++) {
          mn = std::min(mn, h[2 * w]);
          mx = std::max(mx, h[2 * w + 1]);
          lat.push_back((h[2 * w + 1] - h[2 * w]) / 1e3);
        }
        std::sort(lat.begin(), lat.end());
        printf("warps %5d ops %d %-24s span %7.2f us  latency med %6.2f p90 %6.2f max %6.2f us\n", nact, ops,
               names[mode], (mx - mn) / 1e3, lat[lat.size() / 2], lat[lat.size() * 9 / 10], lat.back());
      }
  return 0;
}
