// eval_sparse.cuh -- EXPERIMENT (libsg_exp.so only; measured slower than the product's S0 trie, profiles/r02_v9.txt):
// the evaluation hot path (rows a2-a6; Alg. 7) for high-dimensional,
// low-level grids (cfg5: d = 20, n = 6), enumerating each level vector by its SUPPORT.
//
// At d = 20 and n = 6 every level vector has at most 5 non-zero entries among 20, so the bijection-order
// trie of eval_trie.cuh spends most of its instructions walking level-0 dimensions (28 instructions per
// term, profiles/r01_v6_cfg5_eval_ncu.txt).  Here the basis product is factored through the level-0 hats:
//     prod_t phi_{l_t}(x_t) = S0(x) * prod_{t : l_t > 0} rho_t(l_t),   S0 = prod_t phi_0(x_t),
//     rho_t(v) = phi_v(x_t) / phi_0(x_t)  in [0, 2^v]  (0 where phi_0(x_t) = 0, where every phi_v vanishes)
// (reading G21), so a level-0 dimension costs nothing, and the level vectors of a sub-trie are enumerated
// by their highest non-zero dimension u and its level v:
//   G(t, B) = sum of the terms of dimensions t..0 with level sum B (l_0 implied, Alg. 3 order: l_t slowest)
//           = [l_1..l_t = 0, l_0 = B]                                    (the sub-trie's first subspace)
//           + sum_{u=1..t} sum_{v=1..B} rho_u(v) G(u-1, B-v)  at subspace offset
//             off(u, B, v) = C(B+u, u) - C(B-v+u, u)   (the subspaces with l_t..l_{u+1} = 0, l_u < v come
//             first: sum_{v'<v} C(B-v'+u-1, u-1), hockey stick)
// and the leaves (v = B) are one gather and one FMA each.  In-subspace index (Alg. 5 digit order, dimension
// 0 most significant): dimension u's v-digit cell k_u(v) sits at bit J - B (the levels of the dimensions
// above u sum to J - B).  The subspace base advances in the bijection order exactly as in the layout, so
// gp2idx is never evaluated.
//
// Per query the kernel keeps rho_t(v) for v = 1..NM-1 in shared memory ([v-1][t][lane]), each word carrying
// the cell digit k_t(v) (v <= 5 bits) in its 5 low mantissa bits (reading G21: a relative perturbation below
// 2^-47 per factor), so one 8-byte shared load gives a factor and its digit.
#pragma once
#include "../common.cuh"
#include "../eval_common.cuh"

namespace sg {
namespace sparse {

constexpr int kDigBits = 5;  // digit bits packed into the ratio words (levels <= 5 below NM)

// binomial coefficients C(a, b), a, b < 40, in constant memory: the offsets are warp-uniform, so they are
// read through the constant cache (no L1 data-pipe wavefronts next to the surplus gathers)
constexpr int kBin = 40;
struct BinomTable {
  uint32_t v[kBin][kBin];
  constexpr BinomTable() : v() {
    for (int a = 0; a < kBin; ++a)
      for (int b = 0; b < kBin; ++b) v[a][b] = (b == 0) ? 1u : (a == 0 ? 0u : v[a - 1][b - 1] + v[a - 1][b]);
  }
};
static __constant__ BinomTable c_binom = BinomTable();

template <typename T, int D, int NM, int NT>
struct Sparse {
  static_assert(NM - 1 <= kDigBits, "cell digits of level <= NM-1 must fit the packed bits");
  static constexpr size_t smem_bytes = (size_t)(NM - 1) * D * NT * sizeof(double);

  struct Ctx {
    const T* __restrict__ alpha;
    const double* rho;  // this lane's column: rho[((v-1) * D + t) * NT]
    int J;
  };

  static_assert(D + NM < kBin, "binomial table too small");
  static __device__ __forceinline__ uint32_t C(int a, int b) { return c_binom.v[a][b]; }
  static __device__ __forceinline__ double word(const Ctx& c, int t, int v) { return c.rho[((v - 1) * D + t) * NT]; }
  static __device__ __forceinline__ uint32_t digit(double w) {
    return (uint32_t)__double2loint(w) & ((1u << kDigBits) - 1u);
  }

  // sum of the terms of the sub-trie of dimensions t..0 with level sum B >= 1 under the subspace base b and
  // the partial index P (digits of the dimensions above t), WITHOUT the hat ratios above t
  template <int DEPTH>
  static __device__ double G(const Ctx& c, int t, int B, uint32_t b, uint32_t P) {
    const int sh = c.J - B;  // bit of dimension u's digits (the levels above u sum to J - B)
    const T* base = c.alpha + b;
    // u = 0 (l_1..l_t = 0, l_0 = B: the sub-trie's first subspace) and the leaves u = 1..t, v = B
    // (everything below u is level 0, offset C(B+u, u) - 1): compile-time u, predicated on u <= t, every
    // shared-memory word and every gather issued before the first FMA (one memory round trip per leaf row;
    // a run-time loop waits for each gather in turn)
    double acc = 0.0;
    constexpr int CH = 10;  // leaf rows in chunks of CH (registers)
#pragma unroll
    for (int u0 = 0; u0 < D; u0 += CH) {
      if (u0 <= t) {
        double w[CH];
        T a[CH];
#pragma unroll
        for (int k = 0; k < CH; ++k)
          if (u0 + k < D && u0 + k <= t) w[k] = word(c, u0 + k, B);
#pragma unroll
        for (int k = 0; k < CH; ++k) {
          const int u = u0 + k;
          if (u < D && u <= t)
            a[k] = __ldg(base + (u == 0 ? 0u : (C(B + u, u) - 1u) << c.J) + (P | (digit(w[k]) << sh)));
        }
#pragma unroll
        for (int k = 0; k < CH; ++k)
          if (u0 + k < D && u0 + k <= t) acc = fma((double)a[k], w[k], acc);
      }
    }
    if constexpr (DEPTH > 1) {
      // internal nodes: u = 1..t, v = 1..B-1, then the sub-trie (u-1, B-v)
      for (int v = 1; v < B; ++v) {
        for (int u = 1; u <= t; ++u) {
          const double wu = word(c, u, v);
          const uint32_t off = (C(B + u, u) - C(B - v + u, u)) << c.J;
          acc = fma(G<DEPTH - 1>(c, u - 1, B - v, b + off, P | (digit(wu) << sh)), wu, acc);
        }
      }
    }
    return acc;
  }
};

// One launch evaluates the level groups 0..n-1 for every query (one thread per query, Morton order via
// perm).  goff[j] = index3(j), the offset of group j.
struct GroupOffsets {
  uint32_t off[16];
};

template <typename T, int D, int NM, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB)
    k_eval_sparse(const T* __restrict__ alpha, const T* __restrict__ x, const uint32_t* __restrict__ perm, uint32_t m,
                  int n, GroupOffsets go, T* __restrict__ y) {
  using SP = Sparse<T, D, NM, NT>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  double* sm = reinterpret_cast<double*>(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t q = blockIdx.x * NT + tid;
  const bool active = q < m;
  const uint32_t src = active ? (perm ? perm[q] : q) : 0u;
  // ---- a2: level-0 hats (S0) and the ratio words of every dimension and level 1..NM-1
  bool bad = false;
  double s0 = 1.0;
  for (int t = 0; t < D; ++t) {
    const double xt = active ? (double)x[(size_t)src * D + t] : 0.5;
    bad |= isnan(xt);
    uint32_t c0;
    const double f0 = hat_cell<double>(xt, 0, c0);
    s0 *= f0;
    const double r0 = f0 > 0.0 ? 1.0 / f0 : 0.0;
#pragma unroll
    for (int v = 1; v < NM; ++v) {
      uint32_t cell;
      const double fv = hat_cell<double>(xt, v, cell);
      const long long bits = (__double_as_longlong(fv * r0) & ~((1ll << kDigBits) - 1)) | (long long)cell;
      sm[((v - 1) * D + t) * NT + tid] = __longlong_as_double(bits);
    }
  }
  // (no barrier: every lane reads only its own shared-memory column)
  typename SP::Ctx c;
  c.alpha = alpha;
  c.rho = sm + tid;
  double res = (double)__ldg(alpha + go.off[0]);  // group 0: the single all-zero level vector
  for (int j = 1; j < n; ++j) {
    c.J = j;
    res += SP::template G<NM - 1>(c, D - 1, j, go.off[j], 0u);
  }
  if (active) y[src] = bad ? T(NAN) : (T)(res * s0);
}

}  // namespace sparse
}  // namespace sg

namespace sg {
namespace sparse {
template <typename T, int D, int NM, int NT, int MINB>
sg_status launch(const Layout& L, const T* alpha, const T* x, const uint32_t* perm, uint64_t m, T* y,
                 cudaStream_t s) {
  if (L.n > NM || L.d != D) return cuda_fail(cudaErrorInvalidValue, "k_eval_sparse: shape");
  auto kern = k_eval_sparse<T, D, NM, NT, MINB>;
  const size_t smem = Sparse<T, D, NM, NT>::smem_bytes;
  const int pct = (int)((smem * MINB * 100 + 227 * 1024 - 1) / (227 * 1024)) + 1;
  static std::atomic<uint64_t> attr_done{0};
  const sg_status st = set_smem_attr(kern, attr_done, smem, pct, "cudaFuncSetAttribute(k_eval_sparse)");
  if (st != SG_OK) return st;
  GroupOffsets go{};
  for (int j = 0; j < L.n; ++j) go.off[j] = (uint32_t)L.off[j];
  const unsigned blocks = (unsigned)((m + NT - 1) / NT);
  kern<<<blocks, NT, smem, s>>>(alpha, x, perm, (uint32_t)m, L.n, go, y);
  return launched("k_eval_sparse", (const void*)kern);
}
}  // namespace sparse
}  // namespace sg
