// l1_order.cu -- microbenchmark (not part of libsg): does an L1 hit wait for
// an L1 miss issued just before it (in-order completion of global loads)?
// One warp per SM.  Reports the cycles until a hit's value is usable, with
// and without an outstanding L2-resident miss issued immediately before it.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l1o l1_order.cu && ./l1o
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k(const double* __restrict__ hot, const double* __restrict__ cold, int with_miss, int iters,
                  unsigned long long* out, double* sink) {
  const int lane = threadIdx.x;
  double acc = 0;
  // warm the hot line into L1
  acc += __ldg(hot + lane);
  unsigned long long tot = 0;
  for (int it = 0; it < iters; ++it) {
    // a different cold line each iteration (L2-resident after the first kernel, L1 miss)
    const double* cp = cold + ((size_t)(blockIdx.x * iters + it) * 64 + lane) % (1u << 22);
    double x = 0, y;
    unsigned long long t0 = clock64();
    if (with_miss) asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(x) : "l"(cp) : "memory");
    asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(y) : "l"(hot + ((lane + it) & 31)) : "memory");
    asm volatile("add.f64 %0, %0, %1;" : "+d"(acc) : "d"(y));  // waits for y only
    unsigned long long t1 = clock64();
    tot += t1 - t0;
    asm volatile("add.f64 %0, %0, %1;" : "+d"(acc) : "d"(x));
  }
  if (lane == 0) out[blockIdx.x] = tot / iters;
  if (acc == 12345.0) sink[0] = acc;
}

int main() {
  double *hot, *cold, *sink;
  unsigned long long* out;
  cudaMalloc(&hot, 4096);
  cudaMalloc(&cold, (size_t)8 << 22);
  cudaMemset(hot, 0, 4096);
  cudaMemset(cold, 0, (size_t)8 << 22);
  cudaMalloc(&sink, 8);
  cudaMalloc(&out, 148 * 8);
  unsigned long long h[148];
  for (int rep = 0; rep < 2; ++rep)
    for (int wm = 0; wm < 2; ++wm) {
      k<<<148, 32>>>(hot, cold, wm, 200, out, sink);
      cudaDeviceSynchronize();
      cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
      double s = 0;
      for (int i = 0; i < 148; ++i) s += h[i];
      if (rep) printf("hit latency %s a preceding miss: %.1f cycles\n", wm ? "WITH" : "without", s / 148);
    }
  return 0;
}
