// eval_gen.cuh -- the evaluation path for every grid shape without a specialised instantiation
// (rows a2-a6; Alg. 7): the bijection-order trie of eval_trie.cuh with the level group
// j a RUN-TIME value, so one instantiation per dimension D serves every level n <= NMX (=12).
//
// Same enumeration (Alg. 3 order; warp-uniform running subspace base) and
// the same blocks over the I = min(D, 4) innermost dimensions (C(R+I-1, I-1) consecutive subspaces
// with l_0 implied, R compile-time), so per term the index is still ONE 3-input logic op
//     index1' = (C''[s] & M_row) | X_row
// The price of a run-time j is paid per block and per row, not per term:
//   * the subspace offset c * 2^j can no longer be a load immediate: the row pointer
//     rp = &alpha[b + P + (c_row - q_row) 2^j] is formed once per row (q_row = l_2 + l_3) and
//     C''[s] = C'[s] | (s << j) carries the rest (s - q_row = l_1, the term's rank in its row;
//     bits >= j are free in C'[s]), so the in-row offset still rides in the one LOP3;
//   * the row mask M_row = ~0 << (l_2 + l_3 + sigma) and the dimension-2/3 digits are shifted by
//     run-time amounts (sigma = j - R).
// Cells k_t(l) = K_t >> (NMX-1-l), K_t = clamp(floor(2^{NMX-1} x_t)) (exact for l <= NMX-1);
// hat values 2 min(u, 1-u) (reading G7); dimensions 0, 1 in registers, 2, 3 and I in shared memory,
// dimensions > I by exact doubling along their loops (2u or 2 - 2u, out-of-cube queries flagged and written
// as 0), a CTA barrier per step of the top loop -- as in eval_trie.cuh.
#pragma once
#include "common.cuh"
#include "eval_common.cuh"

namespace sg {
namespace gen {

constexpr int NMX = 12;  // level bound of the generic kernels: n <= 12

template <typename T, int D, int NT>
struct GTrie {
  static constexpr int NM = NMX;
  static constexpr int I = D < 4 ? D : 4;  // inner (block) dimensions
  static constexpr int O = D - I;          // outer (trie) dimensions
  static constexpr int SM_IN = 2 * NM;     // hat tables of dimensions 2, 3
  static constexpr int SM_PH = O > 0 ? NM : 0;
  static constexpr int SM_X = O > 1 ? O - 1 : 0;
  static constexpr int xrow(int t) { return t - I - 1; }
  static constexpr size_t smem_bytes = (size_t)(SM_IN + SM_PH + SM_X) * NT * sizeof(T);

  struct Ctx {
    const T* __restrict__ alpha;
    const T* phs;  // this lane's column of the hat tables (dims 2, 3, I)
    const T* xs;   // this lane's column of the x table of dimensions > I
    T ph[I < 2 ? I : 2][NM];  // hat values of dimensions 0, 1
    uint32_t K[D];
    double res;
    uint32_t b;  // running subspace base (elements), warp-uniform
    int J;       // current level group (run time)
    int vlo, vhi;  // levels l_{D-1} of the top trie loop this launch evaluates (a part of a sharded grid)
  };

  static constexpr uint32_t cnt(int R) {  // subspaces per block = C(R+I-1, I-1)
    uint32_t c = 1;
    for (int k = 1; k <= I - 1; ++k) c = c * (uint32_t)(R + k) / (uint32_t)k;
    return c;
  }
  static __device__ __forceinline__ uint32_t lowmask(int k) { return k >= 32 ? 0xffffffffu : ((1u << k) - 1u); }

  // block of budget R (compile time) in group c.J (run time)
  template <int R>
  static __device__ __forceinline__ void block(Ctx& c, uint32_t P, T prod) {
    const int J = c.J;
    const int SG = J - R;  // sigma = sum of the outer levels
    const T* base = c.alpha + c.b + P;
    uint32_t k0, k1, k2, k3;  // opaque copies: keep the per-block cell work inside the trie
    asm volatile("mov.b32 %0, %1;" : "=r"(k0) : "r"(c.K[0]));
    asm volatile("mov.b32 %0, %1;" : "=r"(k1) : "r"(c.K[I > 1 ? 1 : 0]));
    asm volatile("mov.b32 %0, %1;" : "=r"(k2) : "r"(c.K[I > 2 ? 2 : 0]));
    asm volatile("mov.b32 %0, %1;" : "=r"(k3) : "r"(c.K[I > 3 ? 3 : 0]));
    // C''[s] = (k_0(R-s) << (s+SG)) | (k_1 digits at level s, shifted by SG) | (s << J)
    const uint32_t K0J = k0 >> (NM - 1 - J);
    uint32_t Cs[R + 1];
#pragma unroll
    for (int s = 0; s <= R; ++s) {
      const uint32_t hi = K0J & ~lowmask(s + SG);
      const uint32_t lo = (I > 1) ? (k1 >> (NM - 1 - s - SG)) : 0u;
      Cs[s] = hi | lo | ((uint32_t)s << J);
    }
    T ph2[R + 1];
#pragma unroll
    for (int l = 0; l <= R; ++l) ph2[l] = (I >= 3) ? c.phs[(0 * NM + l) * NT] : T(1);
    T acc = T(0);
    constexpr int R3 = (I >= 4) ? R : 0;
    int crow = 0;  // compile-time after unrolling: rank of the row's first term inside the block
#pragma unroll
    for (int l3 = 0; l3 <= R3; ++l3) {
      const uint32_t X3 = (I >= 4) ? ((k3 >> (NM - 1 - l3 - SG)) & ~lowmask(SG)) : 0u;
      const int R2 = (I >= 3) ? R - l3 : 0;
      T acc3 = T(0);
#pragma unroll
      for (int l2 = 0; l2 <= R2; ++l2) {
        uint32_t Xr = (I >= 3) ? (((k2 >> (NM - 1 - l2 - l3 - SG)) & ~lowmask(l3 + SG)) | X3) : X3;
        const uint32_t M = ~lowmask(l2 + l3 + SG);
        const int R1 = (I >= 2) ? R - l3 - l2 : 0;
        // row pointer: &alpha[b + P + (crow - l2 - l3) 2^J]; the term adds (s << J) + index1 through C''[s]
        const T* rp = base + (size_t)(((uint32_t)(crow - l2 - l3)) << J);
        T acc2 = T(0);
#pragma unroll
        for (int l1 = 0; l1 <= R1; ++l1) {
          const int s = l1 + l2 + l3;
          const int l0 = R - s;
          uint32_t V;
          asm("lop3.b32 %0, %1, %2, %3, 0xEA;" : "=r"(V) : "r"(Cs[s]), "r"(M), "r"(Xr));
          const T a = __ldg(rp + V);
          if (I >= 2) acc2 = fma(a * c.ph[0][l0], c.ph[I > 1 ? 1 : 0][l1], acc2);
          else acc2 = fma(a, c.ph[0][l0], acc2);
        }
        crow += R1 + 1;
        acc3 = (I >= 3) ? fma(acc2, ph2[l2], acc3) : acc2;
      }
      if constexpr (I >= 4) acc = fma(acc3, c.phs[(1 * NM + l3) * NT], acc);
      else acc = acc3;
    }
    c.res = fma((double)acc, (double)prod, c.res);
    c.b += cnt(R) << J;
  }

#define SG_GEN_CASE(r) \
  case r:              \
    block<r>(c, P, prod); \
    break;
  static __device__ __forceinline__ void leaf(Ctx& c, int R, uint32_t P, T prod) {
    switch (R) {
      SG_GEN_CASE(0) SG_GEN_CASE(1) SG_GEN_CASE(2) SG_GEN_CASE(3)
      SG_GEN_CASE(4) SG_GEN_CASE(5) SG_GEN_CASE(6) SG_GEN_CASE(7)
      SG_GEN_CASE(8) SG_GEN_CASE(9) SG_GEN_CASE(10) SG_GEN_CASE(11)
      default: break;
    }
  }
#undef SG_GEN_CASE

  // 2 min(u, 1-u) for u in [0, 1] as 2u or 2 - 2u (exact; queries outside the cube are written as 0, reading G8)
  static __device__ __forceinline__ T hat_u(T u) {
    const T t = u + u;
    return t < T(1) ? t : T(2) - t;
  }
  static __device__ __forceinline__ T dbl_u(T u) {
    u = u + u;
    return u >= T(1) ? u - T(1) : u;
  }

  // tail of dimension I at run-time budget B: the blocks R = RT .. 0 merged into one basic block
  template <int RT>
  static __device__ __forceinline__ void inner_tail(Ctx& c, int B, uint32_t P, T prod) {
    if constexpr (RT >= 0) {
      if (RT <= B) {
        const int lt = B - RT;
        const T ph = c.phs[(SM_IN + lt) * NT];
        const uint32_t kt = c.K[I] >> (NM - 1 - lt);
        block<RT>(c, P | (kt << (c.J - B)), prod * ph);
      }
      inner_tail<RT - 1>(c, B, P, prod);
    }
  }

  // node at dimension t >= I with run-time budget B: a run-time loop over l_t
  template <int t>
  static __device__ __forceinline__ void node(Ctx& c, int B, uint32_t P, T prod) {
    const int SG = c.J - B;
    if constexpr (t == I) {
      constexpr int kTail = 3;
      for (int lt = 0; lt < B - kTail; ++lt) {
        const T ph = c.phs[(SM_IN + lt) * NT];
        const uint32_t kt = c.K[I] >> (NM - 1 - lt);
        leaf(c, B - lt, P | (kt << SG), prod * ph);
      }
      inner_tail<kTail>(c, B, P, prod);
    } else {
      T u = c.xs[xrow(t) * NT];
      int lt0 = 0, lt1 = B;
      if (t == D - 1) {  // the top loop: a part of a sharded grid may start / end inside it
        lt0 = c.vlo;
        lt1 = c.vhi < B ? c.vhi : B;
        for (int k = 0; k < lt0; ++k) u = dbl_u(u);
      }
      for (int lt = lt0; lt <= lt1; ++lt) {
        // the top loop: a CTA barrier per level step keeps the CTA's warps in step through the enumeration
        // (they share L1 lines; eval_trie.cuh Knobs::SYNC); uniform: every thread runs the same trie
        if constexpr (t == D - 1 && NT > 32) __syncthreads();
        const uint32_t kt = c.K[t] >> (NM - 1 - lt);
        node<t - 1>(c, B - lt, P | (kt << SG), prod * hat_u(u));
        u = dbl_u(u);
      }
    }
  }
};

template <typename T, int D, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB)
    k_eval_gen(const T* __restrict__ alpha, const T* __restrict__ x, const uint32_t* __restrict__ perm, uint32_t m,
               int n, T* __restrict__ y, int j0, int v0, int j1, int v1, uint32_t b0, int accumulate) {
  using TR = GTrie<T, D, NT>;
  constexpr int I = TR::I, NM = TR::NM;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* sm = reinterpret_cast<T*>(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t q = blockIdx.x * NT + tid;
  const bool active = q < m;
  const uint32_t src = active ? (perm ? perm[q] : q) : 0u;
  typename TR::Ctx c;
  c.alpha = alpha;
  c.phs = sm + tid;
  c.xs = sm + (TR::SM_IN + TR::SM_PH) * NT + tid;
  bool bad = false, outside = false;
  const T fine = (T)(1u << (NM - 1));
#pragma unroll
  for (int t = 0; t < D; ++t) {
    const T xt = active ? x[(size_t)src * D + t] : T(0.5);
    bad |= isnan(xt);
    outside |= !(xt >= T(0) && xt <= T(1));
    T kf = floor(xt * fine);
    kf = kf > T(0) ? kf : T(0);
    kf = kf < fine - T(1) ? kf : fine - T(1);
    c.K[t] = (uint32_t)kf;
    if (t <= I) {
#pragma unroll
      for (int l = 0; l < NM; ++l) {
        uint32_t cell;
        const T h = hat_cell<T>(xt, l, cell);
        if (t < 2) c.ph[t < 2 ? t : 0][l] = h;
        else if (t < I) sm[((t - 2) * NM + l) * NT + tid] = h;
        else sm[(TR::SM_IN + l) * NT + tid] = h;
      }
    } else {
      sm[(TR::SM_IN + TR::SM_PH + TR::xrow(t)) * NT + tid] = xt;
    }
  }
  c.res = 0.0;
  c.b = b0;  // index3(j0) + the subspaces of group j0 before level l_{D-1} = v0 (times 2^j0)
  // level groups in the bijection order; a sharded grid's part (sg_evaluate_part) covers
  // the groups j0..j1, starting at l_{D-1} = v0 in group j0 and ending at l_{D-1} = v1 in group j1
  for (int J = j0; J <= j1 && J < n; ++J) {
    c.J = J;
    c.vlo = J == j0 ? v0 : 0;
    c.vhi = J == j1 ? v1 : J;
    if constexpr (TR::O == 0) TR::leaf(c, J, 0u, T(1));  // one block per group
    else TR::template node<D - 1>(c, J, 0u, T(1));
  }
  if (active) {
    double r = c.res;
    if (accumulate) r += (double)y[src];
    y[src] = bad ? T(NAN) : (outside ? T(0) : (T)r);
  }
}

// Part of the groups: j0..j1 with l_{D-1} in [v0, ..] in group j0 and [.., v1] in group j1 (D >= 6; whole groups
// otherwise), the running base starting at b0; accumulate adds to y.  Default: the whole grid.
template <typename T, int D>
sg_status launch_gen(const T* alpha, const T* x, const uint32_t* perm, uint64_t m, int n, T* y, cudaStream_t s,
                     int j0 = 0, int v0 = 0, int j1 = 64, int v1 = 64, uint32_t b0 = 0, int accumulate = 0) {
  constexpr int NT = 128, MINB = 3;
  using TR = GTrie<T, D, NT>;
  auto kern = k_eval_gen<T, D, NT, MINB>;
  const size_t smem = TR::smem_bytes;
  const int pct = (int)((smem * MINB * 100 + 227 * 1024 - 1) / (227 * 1024)) + 1;
  static std::atomic<uint64_t> attr_done{0};
  const sg_status st = set_smem_attr(kern, attr_done, smem, pct, "cudaFuncSetAttribute(k_eval_gen)");
  if (st != SG_OK) return st;
  const unsigned blocks = (unsigned)((m + NT - 1) / NT);
  kern<<<blocks, NT, smem, s>>>(alpha, x, perm, (uint32_t)m, n, y, j0, v0, j1, v1, b0, accumulate);
  return launched("k_eval_gen", (const void*)kern);
}

}  // namespace gen
}  // namespace sg
