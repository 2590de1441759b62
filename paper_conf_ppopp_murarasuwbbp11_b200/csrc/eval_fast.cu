// eval_fast.cu -- the evaluation hot path (rows a2-a6; Alg. 7),
// specialised on the dimension D (compile time) and a level bound NM >= n.
//
// Work decomposition: one query per thread, queries Morton-ordered (row a1)
// so that the 32 lanes of a warp -- and the warps of a CTA -- fall into the
// same or neighbouring cells of every subspace and their surplus gathers
// share L1/L2 sectors.  Every lane runs the SAME enumeration of level vectors
// (warp-uniform control flow, the B200 analogue of the paper's block-shared
// level vector), in the bijection order: group j = 0..n-1, inside a
// group the Alg. 3 order (l_{D-1} slowest, l_1 fastest, l_0
// implied), so the subspace base offset index3 + index2 simply advances by
// 2^j per subspace (Alg. 7 "index2 += 2^j"); gp2idx is never evaluated.
//
// The enumeration is a trie over dimensions D-1 .. 3 (template recursion,
// runtime loop over l_t at every level) whose leaves are "blocks": all
// (l_2, l_1) with l_0 + l_1 + l_2 = R for the remaining budget R.  A block is
// fully unrolled per R (switch), so the 1D quantities of dimensions 0..2 --
// hat values phi_t[l] and finest cells K_t -- live in registers with
// compile-time indices; dimensions >= 3 keep their hat values in shared
// memory ([t][l][lane], conflict-free) and are touched once per trie node.
//
// Per term: in-subspace index (Alg. 5 digit order, dimension 0 most
// significant) from three masked/shifted cells OR-ed together, one read-only
// gather, one DMUL + one DFMA (Horner over l_1, then l_2, then the trie
// prefix product).  Cells: k_t(l) = K_t >> (NM-1-l) with
// K_t = clamp(floor(2^{NM-1} x_t)) (exact).
#include "common.cuh"
#include "eval_common.cuh"

namespace sg {

namespace {

constexpr int kThreads = 128;

template <typename T, int D, int NM>
struct Ctx {
  const T* __restrict__ alpha;
  const T* phis;  // shared: [(D-3)][NM][kThreads] hat values of dims >= 3 (this lane's column)
  uint32_t K[D];  // finest cell per dimension
  T ph0[NM], ph1[NM], ph2[NM];
  double res;  // fp64 also for fp32 storage (long sequential sum over the blocks)
  uint64_t b;  // base offset index3 + index2 of the next subspace (warp-uniform)
  int j;       // current level group
};

// ---- one block: all (l2, l1) with l0 = R - l1 - l2, in Alg. 3 order --------
template <typename T, int D, int NM, int R>
__device__ __forceinline__ void block(Ctx<T, D, NM>& c, int s3, uint32_t P3, T prod3) {
  // per-lane address of the block's first surplus for this lane's digits of
  // dimensions >= 3; per term the in-block offset (< 2^32) is shifted by s3
  const T* pl = c.alpha + (c.b + P3);
  asm volatile("mov.b64 %0, %0;" : "+l"(pl));
  // Opaque per-block copies of the finest cells: the in-block offsets depend
  // only on (K0, K1, K2) and compile-time constants, and without this the
  // compiler hoists all C(NM+2, 3) of them out of the trie and spills them.
  uint32_t k0, k1, k2;
  asm volatile("mov.b32 %0, %1;" : "=r"(k0) : "r"(c.K[0]));
  asm volatile("mov.b32 %0, %1;" : "=r"(k1) : "r"(c.K[1]));
  asm volatile("mov.b32 %0, %1;" : "=r"(k2) : "r"(c.K[D > 2 ? 2 : 0]));
  const uint32_t K0R = k0 >> (NM - 1 - R);
  T acc = T(0);
#pragma unroll
  for (int l2 = 0; l2 <= R; ++l2) {
    const uint32_t X2 = (D > 2) ? (k2 >> (NM - 1 - l2)) : 0u;
    T acc1 = T(0);
#pragma unroll
    for (int l1 = 0; l1 <= R - l2; ++l1) {
      const int l0 = R - l2 - l1;
      const uint32_t cpos = (uint32_t)(l2 * (R + 1) - (l2 * (l2 - 1)) / 2 + l1);  // rank inside the block
      const uint32_t X0 = K0R & ~((1u << (l1 + l2)) - 1u);                       // k_0(l0) << (l1+l2)
      const uint32_t X1 = (k1 >> (NM - 1 - l1 - l2)) & ~((1u << l2) - 1u);      // k_1(l1) << l2
      const uint32_t off = (cpos << R) | X0 | X1 | X2;
      const T a = __ldg(pl + (off << s3));
      acc1 = fma(a * c.ph0[l0], c.ph1[l1], acc1);
    }
    acc = (D > 2) ? fma(acc1, c.ph2[l2], acc) : acc1;
    asm volatile("" ::: "memory");  // keep at most one row of gathers in flight (register budget)
  }
  c.res = fma((double)acc, (double)prod3, c.res);
  c.b += (uint64_t)((R + 1) * (R + 2) / 2) << c.j;
}

#define SG_BLOCK_CASE(r) \
  case r:                \
    if constexpr (r < NM) block<T, D, NM, r>(c, s3, P3, prod3); \
    break;

template <typename T, int D, int NM>
__device__ __forceinline__ void bottom(Ctx<T, D, NM>& c, int R, int s3, uint32_t P3, T prod3) {
  switch (R) {
    SG_BLOCK_CASE(0) SG_BLOCK_CASE(1) SG_BLOCK_CASE(2) SG_BLOCK_CASE(3)
    SG_BLOCK_CASE(4) SG_BLOCK_CASE(5) SG_BLOCK_CASE(6) SG_BLOCK_CASE(7)
    SG_BLOCK_CASE(8) SG_BLOCK_CASE(9) SG_BLOCK_CASE(10) SG_BLOCK_CASE(11)
    SG_BLOCK_CASE(12) SG_BLOCK_CASE(13) SG_BLOCK_CASE(14) SG_BLOCK_CASE(15)
    default: break;
  }
}
#undef SG_BLOCK_CASE

// ---- trie over dimensions t = D-1 .. 3 (Alg. 3 order: ascending l_t, outer = slower)
template <typename T, int D, int NM, int t>
struct Upper {
  static __device__ __forceinline__ void run(Ctx<T, D, NM>& c, int budget, int suf, uint32_t P, T prod) {
    for (int lt = 0; lt <= budget; ++lt) {
      const T ph = c.phis[((t - 3) * NM + lt) * kThreads];
      const uint32_t Pt = P + ((c.K[t] >> (NM - 1 - lt)) << suf);
      Upper<T, D, NM, t - 1>::run(c, budget - lt, suf + lt, Pt, prod * ph);
    }
  }
};
template <typename T, int D, int NM>
struct Upper<T, D, NM, 2> {
  static __device__ __forceinline__ void run(Ctx<T, D, NM>& c, int budget, int suf, uint32_t P, T prod) {
    bottom<T, D, NM>(c, budget, suf, P, prod);
  }
};

template <typename T, int D, int NM>
__global__ void __launch_bounds__(kThreads, 2)
    k_eval_fast(const T* __restrict__ alpha, const T* __restrict__ x, const uint32_t* __restrict__ perm, uint32_t m,
                int n, T* __restrict__ y) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* phis = reinterpret_cast<T*>(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t q = blockIdx.x * kThreads + tid;
  const bool active = q < m;
  const uint32_t src = active ? (perm ? perm[q] : q) : 0u;

  Ctx<T, D, NM> c;
  c.alpha = alpha;
  c.phis = phis + tid;
  // ---- a2: finest cells and hat values of every dimension and level
  bool bad = false;
  const T fine = (T)(1u << (NM - 1));
#pragma unroll
  for (int t = 0; t < D; ++t) {
    const T xt = active ? x[(size_t)src * D + t] : T(0.5);
    bad |= isnan(xt);
    T kf = floor(xt * fine);
    kf = kf > T(0) ? kf : T(0);
    kf = kf < fine - T(1) ? kf : fine - T(1);
    c.K[t] = (uint32_t)kf;
#pragma unroll
    for (int l = 0; l < NM; ++l) {
      uint32_t cell;
      const T h = hat_cell<T>(xt, l, cell);
      if (t == 0) c.ph0[l] = h;
      else if (t == 1) c.ph1[l] = h;
      else if (t == 2) c.ph2[l] = h;
      else phis[((t - 3) * NM + l) * kThreads + tid] = h;
    }
  }
  if (D < 3) {
#pragma unroll
    for (int l = 0; l < NM; ++l) c.ph2[l] = T(1);
  }
  // (no barrier needed: every lane reads only its own shared-memory column)
  c.res = 0.0;
  c.b = 0;
  for (int j = 0; j < n; ++j) {
    c.j = j;
    Upper<T, D, NM, D - 1>::run(c, j, 0, 0u, T(1));
  }
  if (active) y[src] = bad ? T(NAN) : (T)c.res;
}

template <typename T, int D, int NM>
sg_status launch_t(const T* alpha, const T* x, const uint32_t* perm, uint64_t m, int n, T* y, cudaStream_t s) {
  static_assert(D >= 3, "fast kernel needs D >= 3");
  const size_t smem = (size_t)(D - 3) * NM * kThreads * sizeof(T);
  static std::atomic<uint64_t> attr_done{0};
  sg_status st = set_smem_attr(k_eval_fast<T, D, NM>, attr_done, smem, -1, "cudaFuncSetAttribute(k_eval_fast)");
  if (st != SG_OK) return st;
  const unsigned blocks = (unsigned)((m + kThreads - 1) / kThreads);
  k_eval_fast<T, D, NM><<<blocks, kThreads, smem, s>>>(alpha, x, perm, (uint32_t)m, n, y);
  return launched("k_eval_fast");
}

template <typename T>
sg_status dispatch(int d, int n, const T* alpha, const T* x, const uint32_t* perm, uint64_t m, T* y, cudaStream_t s,
                   bool* handled) {
  *handled = true;
#define SG_FAST(DD, NN) \
  if (d == DD && n <= NN) return launch_t<T, DD, NN>(alpha, x, perm, m, n, y, s);
  SG_FAST(3, 14)
  SG_FAST(5, 8)
  SG_FAST(5, 11)
  SG_FAST(10, 11)
  SG_FAST(20, 6)
#undef SG_FAST
  *handled = false;
  return SG_OK;
}

}  // namespace

sg_status launch_eval_fast(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                           void* y, sg_dtype dt, cudaStream_t s, bool* handled) {
  *handled = false;
  if (m > 0xffffffffull) return SG_OK;
  const int d = g->L.d, n = g->L.n;
  if (dt == SG_F64)
    return dispatch<double>(d, n, (const double*)alpha, (const double*)x, perm, m, (double*)y, s, handled);
  return dispatch<float>(d, n, (const float*)alpha, (const float*)x, perm, m, (float*)y, s, handled);
}

}  // namespace sg
