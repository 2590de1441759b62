// eval_simple.cu -- generic evaluation kernel (Alg. 7), any d <= 32,
// n <= 31, fp64/fp32.  One thread per query; level vectors enumerated in the
// bijection order with Alg. 4 next(), identically in every lane
// (warp-uniform control flow); per term the d hat values and index1 digits
// are recomputed as in Alg. 7.  This is the correctness baseline and the
// fallback for shapes the generic kernel (eval_gen.cuh: d <= 12 or 16, 20; n <= 12) does not cover.
//
// Hat value: phi_{l,i}(x) = max(0, 1 - |2^{l+1} x - i|) is computed as
// 2 * min(u, 1 - u), u = 2^l x - k, k = clamp(floor(2^l x)): the same value
// with no rounding (2^l x and u are exact, 1-u is exact when it is the
// minimum), see DESIGN.md "Exact hat".
#include "common.cuh"
#include "eval_common.cuh"

namespace sg {

namespace {

constexpr int kThreads = 128;

template <typename T>
__global__ void __launch_bounds__(kThreads) k_eval_simple(const Layout* __restrict__ gL, const T* __restrict__ alpha,
                                                          const T* __restrict__ x, const uint32_t* __restrict__ perm,
                                                          uint64_t m, T* __restrict__ y) {
  __shared__ uint64_t cnt[SG_MAX_N];
  __shared__ int dn[2];
  if (threadIdx.x < SG_MAX_N) cnt[threadIdx.x] = gL->cnt[threadIdx.x];
  if (threadIdx.x == 0) {
    dn[0] = gL->d;
    dn[1] = gL->n;
  }
  __syncthreads();
  const int d = dn[0], n = dn[1];
  for (uint64_t q0 = (uint64_t)blockIdx.x * blockDim.x; q0 < m; q0 += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t q = q0 + threadIdx.x;
    const bool active = q < m;
    const uint64_t src = active ? (perm ? (uint64_t)perm[q] : q) : 0;
    T xq[SG_MAX_D];
    bool bad = false;
    for (int t = 0; t < d; ++t) {
      xq[t] = active ? x[src * d + t] : T(0.5);
      bad |= isnan(xq[t]);
    }
    int32_t l[SG_MAX_D + 1];
    double res = 0.0;  // fp64 also for fp32 storage: T sequential terms (reading G13)
    uint64_t base = 0;  // index3 + index2 (Alg. 7 "index2")
    for (int j = 0; j < n; ++j) {
      l[0] = j;  // first(d, j) = (j, 0, ..., 0)   (eq. 3)
      for (int t = 1; t < d; ++t) l[t] = 0;
      const uint64_t cj = cnt[j];
      for (uint64_t k = 0; k < cj; ++k) {
        uint64_t index1 = 0;
        T prod = T(1);
        for (int t = 0; t < d; ++t) {
          const int lt = l[t];
          uint32_t cell;
          prod *= hat_cell<T>(xq[t], lt, cell);
          index1 = (index1 << lt) + cell;
        }
        res += (double)prod * (double)__ldg(alpha + base + index1);
        base += (uint64_t)1 << j;
        if (k + 1 < cj) {  // Alg. 4 next(l); never applied to last(d, j) (reading G5)
          int t = 0;
          while (l[t] == 0) ++t;
          const int lt = l[t];
          l[t] = 0;
          l[0] = lt - 1;
          l[t + 1] += 1;
        }
      }
    }
    if (active) y[src] = bad ? T(NAN) : (T)res;
  }
}

}  // namespace

sg_status launch_eval_simple(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                             void* y, sg_dtype dt, cudaStream_t s) {
  uint64_t blocks = (m + kThreads - 1) / kThreads;
  if (blocks > (uint64_t)kNumSMs * 64) blocks = (uint64_t)kNumSMs * 64;
  if (dt == SG_F64)
    k_eval_simple<double><<<(unsigned)blocks, kThreads, 0, s>>>(g->d_L, (const double*)alpha, (const double*)x, perm,
                                                                m, (double*)y);
  else
    k_eval_simple<float><<<(unsigned)blocks, kThreads, 0, s>>>(g->d_L, (const float*)alpha, (const float*)x, perm, m,
                                                               (float*)y);
  return launched("k_eval_simple", dt == SG_F64 ? (const void*)k_eval_simple<double> : (const void*)k_eval_simple<float>);
}

}  // namespace sg
