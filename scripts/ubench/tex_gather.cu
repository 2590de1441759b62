// tex_gather.cu -- microbenchmark (not part of libsg): cost of one warp-wide 8-byte gather through the
// texture path (tex1Dfetch<int2> on a linear texture, TLD) vs the LSU path (LDG.64), as a function of
// the words / bank pairs the 32 lanes touch (same patterns as l1_gather.cu), L1-resident 32 KB buffer.
// Reports SM cycles per warp-request (all SMs busy, 16 warps per SM).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/texg tex_gather.cu && /tmp/texg
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ int pattern(int mode, int lane, int kk) {
  const int s = lane % kk;
  switch (mode) {
    case 0: return s * 4;                  // k words, 4 apart (packed sectors)
    case 1: return s * 16;                 // k words, one per line, same bank pair
    case 2: return s * 16 + (s & 3) * 4;   // k words, one per line, rotating bank pair
    case 3: return lane;                   // coalesced 256 B
    default: return (lane * 97) & 4095;    // 32 scattered words
  }
}

template <bool TEX>
__global__ void k(const double* __restrict__ buf, cudaTextureObject_t tex, int mode, int kk, int iters, double* out,
                  unsigned long long* cyc) {
  const int lane = threadIdx.x & 31;
  int off = pattern(mode, lane, kk);
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  off = (off + (warp & 7) * 512) & 4095;
  double acc = 0;
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    double a[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int idx = (off + u * 512) & 4095;
      if (TEX) {
        int2 v = tex1Dfetch<int2>(tex, idx);
        a[u] = __hiloint2double(v.y, v.x);
      } else {
        a[u] = __ldg(buf + idx);
      }
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) acc += a[u];
    off = off + (acc == 12345.0 ? 1 : 0);
  }
  unsigned long long t1 = clock64();
  if (acc == 1.0) out[0] = acc;
  if (threadIdx.x == 0) atomicAdd(cyc, t1 - t0);
}

int main() {
  double* buf; double* out; unsigned long long* cyc;
  cudaMalloc(&buf, 4096 * 8); cudaMemset(buf, 0, 4096 * 8);
  cudaMalloc(&out, 8); cudaMalloc(&cyc, 8);
  cudaResourceDesc rd = {};
  rd.resType = cudaResourceTypeLinear;
  rd.res.linear.devPtr = buf;
  rd.res.linear.desc = cudaCreateChannelDesc<int2>();
  rd.res.linear.sizeInBytes = 4096 * 8;
  cudaTextureDesc td = {};
  td.readMode = cudaReadModeElementType;
  cudaTextureObject_t tex;
  if (cudaCreateTextureObject(&tex, &rd, &td, nullptr) != cudaSuccess) { printf("tex create failed\n"); return 1; }
  const int threads = 512, blocks = 148, iters = 2000;
  const char* names[] = {"packed", "1/line same-offset", "1/line rotated", "coalesced256B", "scattered32"};
  for (int path = 0; path < 2; ++path)
    for (int mode = 0; mode < 5; ++mode)
      for (int kk : {1, 2, 4, 8, 16, 32}) {
        if (mode >= 3 && kk != 1) continue;
        for (int rep = 0; rep < 2; ++rep) {
          cudaMemset(cyc, 0, 8);
          cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
          cudaEventRecord(e0);
          if (path) k<true><<<blocks, threads>>>(buf, tex, mode, kk, rep ? iters : 50, out, cyc);
          else k<false><<<blocks, threads>>>(buf, tex, mode, kk, rep ? iters : 50, out, cyc);
          cudaEventRecord(e1); cudaEventSynchronize(e1);
          if (!rep) continue;
          float ms; cudaEventElapsedTime(&ms, e0, e1);
          unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
          const double reqs_per_sm = (double)(threads / 32) * iters * 8;
          printf("%s %-20s k=%2d  cycles/request/SM = %.2f   (%.3f ms)\n", path ? "TEX" : "LDG", names[mode], kk,
                 (double)c / blocks / reqs_per_sm, ms);
        }
      }
  cudaError_t e = cudaGetLastError();
  printf("last error: %s\n", cudaGetErrorString(e));
  return 0;
}
