// exp_pw.cuh -- EXPERIMENT (libsg_exp.so only): persistent warps with SM-affine query tiles.  Each warp takes
// 32-query tiles of the Morton order from its SM's contiguous chunk (one counter per SM, then the other SMs'
// chunks), so the warps resident on an SM work on neighbouring queries (L1 sharing) without the idle warps of
// large CTAs.  Same per-query code as the product (eval_query, eval_trie.cuh).
#pragma once
#include "../eval_trie.cuh"

namespace sg {
namespace pw {

template <typename T, int D, int NM, int NT, int MINB, int J0, int J1, class KN>
__global__ void __launch_bounds__(NT, MINB)
    k_eval_trie_pw(const T* __restrict__ alpha, const T* __restrict__ x, const uint32_t* __restrict__ perm,
                   uint32_t m, int n, uint32_t b0, int accumulate, T* __restrict__ y, uint32_t* __restrict__ ctr) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t lane = threadIdx.x & 31u;
  uint32_t smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  const uint32_t tiles = (m + 31u) / 32u;
  uint32_t ch = smid % kNumSMs;
  for (int tried = 0; tried < kNumSMs;) {
    const uint32_t lo = (uint32_t)((uint64_t)tiles * ch / kNumSMs);
    const uint32_t hi = (uint32_t)((uint64_t)tiles * (ch + 1) / kNumSMs);
    uint32_t k = 0;
    if (lane == 0) k = atomicAdd(ctr + ch, 1u);
    k = __shfl_sync(0xffffffffu, k, 0);
    if (lo + k >= hi) {
      ch = (ch + 1 == (uint32_t)kNumSMs) ? 0u : ch + 1;
      ++tried;
      continue;
    }
    trie::eval_query<T, D, NM, NT, J0, J1, KN>(alpha, x, perm, m, n, b0, accumulate, y, reinterpret_cast<T*>(smem_raw),
                                               threadIdx.x, (lo + k) * 32u + lane);
  }
}

inline uint32_t* counters() {
  static uint32_t* p = nullptr;  // experiment build: one device, one stream
  if (!p) cudaMalloc(&p, kNumSMs * sizeof(uint32_t));
  return p;
}

template <typename T, int D, int NM, int NT, int MINB, int J0, int J1, class KN>
sg_status launch_range(const Layout& L, const T* alpha, const T* x, const uint32_t* perm, uint64_t m, T* y,
                       cudaStream_t s) {
  if (J0 >= L.n) return SG_OK;
  using TR = trie::Trie<T, D, NM, NT, KN>;
  auto kern = k_eval_trie_pw<T, D, NM, NT, MINB, J0, J1, KN>;
  const size_t smem = TR::smem_bytes;
  const int pct = (int)((smem * MINB * 100 + 227 * 1024 - 1) / (227 * 1024)) + 1;
  static std::atomic<uint64_t> attr_done{0};
  const sg_status st = set_smem_attr(kern, attr_done, smem, pct, "cudaFuncSetAttribute(k_eval_trie_pw)");
  if (st != SG_OK) return st;
  uint32_t* ctr = counters();
  cudaMemsetAsync(ctr, 0, kNumSMs * sizeof(uint32_t), s);
  const int accumulate = (J0 > 0 || KN::RMIN > 0) ? 1 : 0;
  kern<<<kNumSMs * MINB, NT, smem, s>>>(alpha, x, perm, (uint32_t)m, L.n, (uint32_t)L.off[J0], accumulate, y, ctr);
  return launched("k_eval_trie_pw", (const void*)kern);
}

}  // namespace pw
}  // namespace sg
