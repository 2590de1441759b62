// l1_gather.cu -- microbenchmark (not part of libsg): cost of one warp-wide
// LDG.64 in the L1TEX pipe as a function of the sectors/lines it touches.
// Every warp loops over NI independent loads from an L1-resident 32 KB buffer;
// lane addresses follow a pattern with k distinct sectors.  Reports SM
// cycles per warp-request (all SMs busy, 16 warps per SM).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/l1g l1_gather.cu && /tmp/l1g
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k(const double* __restrict__ buf, int mode, int kk, int iters, double* out, unsigned long long* cyc) {
  const int lane = threadIdx.x & 31;
  int off;  // element offset inside the 32 KB buffer (4096 doubles)
  const int s = lane % kk;
  switch (mode) {
    case 0: off = s * 4; break;                      // k sectors packed in consecutive lines
    case 1: off = s * 16; break;                     // k sectors, one per line, same offset in line (bank-aligned)
    case 2: off = s * 16 + (s & 3) * 4; break;       // k sectors, one per line, rotating offset
    case 3: off = lane; break;                       // coalesced 256 B (8 sectors, 2 lines)
    default: off = (lane * 97) & 4095; break;        // 32 scattered
  }
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  off = (off + (warp & 7) * 512) & 4095;
  double acc = 0;
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const double* p = buf + ((off + it * 0) & 4095);
    double a0 = __ldg(p), a1 = __ldg(p + 0 + 4096 * 0 + 8 * 0 + 0), a2, a3, a4, a5, a6, a7;
    // eight independent requests to distinct (but same-pattern) regions
    a1 = __ldg(buf + ((off + 1024) & 4095));
    a2 = __ldg(buf + ((off + 2048) & 4095));
    a3 = __ldg(buf + ((off + 3072) & 4095));
    a4 = __ldg(buf + ((off + 512) & 4095));
    a5 = __ldg(buf + ((off + 1536) & 4095));
    a6 = __ldg(buf + ((off + 2560) & 4095));
    a7 = __ldg(buf + ((off + 3584) & 4095));
    acc += a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7;
    off = (off + (acc == 12345.0 ? 1 : 0)) ;  // keep loads inside the loop
  }
  unsigned long long t1 = clock64();
  if (acc == 1.0) out[0] = acc;
  if (threadIdx.x == 0) atomicAdd(cyc, t1 - t0);
}

int main() {
  double* buf; double* out; unsigned long long* cyc;
  cudaMalloc(&buf, 4096 * 8); cudaMemset(buf, 0, 4096 * 8);
  cudaMalloc(&out, 8); cudaMalloc(&cyc, 8);
  const int threads = 512, blocks = 148, iters = 2000;
  const char* names[] = {"packed", "1/line same-offset", "1/line rotated", "coalesced256B", "scattered32"};
  for (int mode = 0; mode < 5; ++mode) {
    for (int kk : {1, 2, 4, 8, 16, 32}) {
      if (mode >= 3 && kk != 1) continue;
      cudaMemset(cyc, 0, 8);
      k<<<blocks, threads>>>(buf, mode, kk, 50, out, cyc);
      cudaMemset(cyc, 0, 8);
      cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
      cudaEventRecord(e0);
      k<<<blocks, threads>>>(buf, mode, kk, iters, out, cyc);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
      double avg_cyc = (double)c / blocks;  // per block (thread 0), ~ kernel cycles
      double reqs_per_sm = (double)(threads / 32) * iters * 8;
      printf("%-20s k=%2d  cycles/request/SM = %.2f   (%.3f ms)\n", names[mode], kk, avg_cyc / reqs_per_sm, ms);
    }
  }
  return 0;
}
