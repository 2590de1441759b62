// eval_trie.cuh -- the evaluation hot path (rows a2-a6; Alg. 7), specialised on the
// dimension D, a level bound NM >= n and the level groups of one launch (compile time).
//
// One query per thread; queries Morton-ordered (row a1).  Every lane of a
// warp runs the SAME enumeration of level vectors in the bijection order
// (Alg. 3: l_{D-1} slowest, l_1 fastest, l_0 implied by the group),
// so the subspace base offset index3 + index2 is a warp-uniform running sum
// that advances by 2^j per subspace (Alg. 7 "index2 += 2^j"); gp2idx is never
// evaluated.  The paper's block-shared level vector becomes
// warp-uniform control flow with no barrier.
//
// The level vectors of group j form a trie: dimensions D-1 .. I are runtime
// loops (the "outer" levels), and each leaf is a *block*: every (l_{I-1}, ..,
// l_1) with l_0 = R - l_1 - .. - l_{I-1}, R = j - sum_{t>=I} l_t, i.e.
// C(R+I-1, I-1) subspaces that are consecutive in the layout.  A block is
// fully unrolled for each (j, R) (compile time), so
//   * the subspace offset of its c-th term, c * 2^j, is an immediate of the
//     load instruction;
//   * the in-subspace index (Alg. 5 digit order, dimension 0 most
//     significant) costs ONE 3-input logic op per term:
//       index1 = (C'[s] & M_row) | X_row,    s = l_1 + .. + l_{I-1},
//     where C'[s] = ((k_0(R-s) << s) | (K_1 >> (NM-1-s))) << sigma is
//     computed once per block for s = 0..R (it carries the digits of
//     dimensions 0 and 1, whose levels are tied through l_0 = R - s), M_row
//     clears the bits below (l_2 + .. + l_{I-1} + sigma), and X_row holds the
//     digits of dimensions 2..I-1; the outer dimensions' digits P go into the
//     block's base pointer;
//   * the basis product is Horner over the trie (Alg. 7's product of d hat
//     values): acc_1 += alpha * phi_0(l_0) * phi_1(l_1) per term,
//     one FMA per row / inner level, one per outer trie node.
// Cells: k_t(l) = K_t >> (NM-1-l) with K_t = clamp(floor(2^{NM-1} x_t)),
// exact.  Hat values: 2 min(u, 1-u),
// u = 2^l x - k_t(l), exact (reading G7).  The hat values of dimensions 0, 1
// live in registers, those of dimensions 2, 3 and I in shared memory
// ([row][lane], conflict-free, read once per block / slab / node);
// dimensions > I recompute them along their loop (u <- frac(2u) and the hat
// 2u or 2 - 2u, exact for x in [0,1]; a query with a coordinate outside the
// cube is 0, reading G8).
#pragma once
#include "common.cuh"
#include "eval_common.cuh"

namespace sg {
namespace trie {

// Compile-time knobs of an instantiation.  The defaults are the configuration measured best at
// cfg3 (experiments recorded under profiles/).
struct Knobs {
  // level-0 suffix products and budget-1 closed forms for outer sub-tries (pays at high d: cfg5)
  static constexpr bool S0 = false;
  // experiment builds only (csrc/exp): gather only -- every hat value 1, no hat table read, the same
  // surplus gathers, addresses and Horner adds (the memory ceiling of the access stream)
  static constexpr bool GO = false;
  // dimension-3 hat value read once per slab (l_3) instead of a per-block register array (fewer
  // live registers, the same number of shared-memory reads)
  static constexpr bool LZ3 = false;
  // dimension I: sub-tries of budget <= FULL emitted straight-line; otherwise a loop whose last
  // TAIL + 1 (small) blocks are merged into one basic block (more surplus loads in flight)
  static constexpr int FULL = 4;
  static constexpr int TAIL = 3;
  // block budgets R this launch evaluates (the others only advance the running subspace base):
  // a group can be split into launches by R, so that the launch of the many small blocks needs
  // the register hat tables of dimensions 0, 1 only up to level RMAX (fewer registers, more warps)
  // and the launch of the few large ones prunes every sub-trie of budget < RMIN
  static constexpr int RMIN = 0;
  static constexpr int RMAX = 64;
  // hat values of dimensions 2, 3 in registers (levels < PHN) instead of shared-memory rows read per
  // block: no LDS on the L1 data pipe, more live registers (for launches with a small RMAX)
  static constexpr bool H23 = false;
  // products phi_0(r - l1) phi_1(l1), r <= RMAX, in registers instead of the tables of dimensions 0, 1:
  // one FMA per term instead of a multiply and an FMA (for launches with a small RMAX)
  static constexpr bool D01 = false;
  // inner (block) dimensions: blocks over dimensions 0..INNER-1 (smaller blocks and per-block register
  // arrays with INNER = 3; dimension 3 then becomes the innermost trie loop)
  static constexpr int INNER = 4;
  // the block table C'[s] from a per-query, per-group table C_J[u] (u = s + sigma, compile-time index)
  // computed once per group, instead of R+1 shift/logic pairs per block
  static constexpr bool CST = false;
  // RMIN prunes trie nodes (sub-tries of level sum < RMIN) but does not filter blocks: the complement of
  // a launch with a larger INNER and RMAX = RMIN - 1 (whose blocks are exactly those sub-tries)
  static constexpr bool RMIN_NODES_ONLY = false;
  // experiment builds only: shared-memory hat rows of the block dimensions 2..INNER-1 for all NM levels
  // (r02 v8) instead of the RMAX + 1 levels a block can read (a launch of small blocks then takes
  // 18 KB less shared memory per CTA, and the SM keeps that much more L1 for the surplus gathers)
  static constexpr bool TAB_ALL = false;
  // level-0 hat values of the block dimensions 2..INNER-1 in registers (read in every block)
  static constexpr bool H0 = false;
  // hat values of dimension I (the innermost trie dimension) by doubling along its level loop, like the
  // dimensions above it, instead of a shared-memory row per level (NM - 1 fewer rows: more L1)
  static constexpr bool IDBL = false;
  // a CTA barrier at every level step of dimension SYNC (< 0: none), keeping the warps of a CTA in step
  // through the enumeration so that they share L1 lines (the trie's control flow is identical in every warp
  // and every thread of the CTA, active or not, runs it: the barrier is uniform)
  static constexpr int SYNC = -1;
};
struct KnobsS0 : Knobs {
  static constexpr bool S0 = true;
};

template <typename T, int D, int NM, int NT, class KN>
struct Trie {
  static constexpr int I = D < KN::INNER ? D : KN::INNER;  // inner (block) dimensions
  static constexpr int O = D - I;          // outer (trie) dimensions
  static constexpr bool S0 = KN::S0, GO = KN::GO, LZ3 = KN::LZ3, H23 = KN::H23 && D >= 4;
  static constexpr bool D01 = KN::D01 && D >= 2;
  static constexpr bool CST = KN::CST;
  // shared memory, [row][lane]: hat values of dimensions 2, 3 (read per block / slab), of
  // dimension I (per dimension-I node), then x of dimensions I+1..D-1
  // levels of the block dimensions' hat rows: a block of budget R <= RMAX reads levels 0..R
  static constexpr int PHB = (KN::TAB_ALL || KN::RMAX + 1 >= NM) ? NM : KN::RMAX + 1;
  static constexpr int SM_IN = (I > 2 ? I - 2 : 0) * PHB;  // hat rows of dimensions 2 .. I-1
  static constexpr bool H0 = KN::H0 && I > 2;
  static constexpr bool IDBL = KN::IDBL && O > 0;
  static constexpr int SM_PH = (O > 0 && !IDBL) ? NM : 0;
  static constexpr int SM_X = IDBL ? O : (O > 1 ? O - 1 : 0);
  static constexpr int xrow(int t) { return IDBL ? t - I : t - I - 1; }
  // S0: suffix products P0[t] = prod_{u <= t} phi_0(x_u), t = I..D-1, so that a
  // sub-trie whose level budget is exhausted (every level of dimensions t..0
  // is 0: one term, one surplus) costs one gather and one FMA instead of a
  // chain of t - I + 1 hat evaluations (matters at high d: cfg5, d = 20)
  static constexpr int SM_S0 = (S0 && O > 0) ? O : 0;
  // S0 (budget-1 sub-tries): rho_u = phi_1(x_u) / phi_0(x_u) in [0, 2] (0 where
  // phi_0 = 0, i.e. x outside (0,1), where phi_1 = 0 too), with the level-1
  // cell k_u(1) in its sign bit; one row per dimension
  static constexpr int SM_RHO = (S0 && O > 0 && NM >= 2) ? D : 0;
  static constexpr size_t smem_bytes = (size_t)(SM_IN + SM_PH + SM_X + SM_S0 + SM_RHO) * NT * sizeof(T);
  static constexpr int kFull = KN::FULL;
  static constexpr int kTail = KN::TAIL;
  static constexpr int RMIN = KN::RMIN, RMAX = KN::RMAX;
  static constexpr int PHN = NM < RMAX + 1 ? NM : RMAX + 1;  // levels of the register hat tables

  struct Ctx {
    const T* __restrict__ alpha;
    const T* phs;  // this lane's column of the hat tables (dims 2, 3, I)
    const T* xs;   // this lane's column of the x table of dimensions > I
    const T* s0;   // S0: this lane's column of the level-0 suffix products
    const T* rho;  // S0: this lane's column of the signed level-1/level-0 hat ratios
    T ph[I < 2 ? I : 2][D01 ? 1 : PHN];  // hat values of dimensions 0, 1 (registers), levels < PHN
    T d01[D01 ? PHN * (PHN + 1) / 2 : 1];  // D01: phi_0(r - l1) phi_1(l1) at index r (r + 1) / 2 + l1
    uint32_t ct[CST ? NM : 1];             // CST: C_J[u] = (k_0 digits of level J above bit u) | (K_1 >> (NM-1-u))
    T ph23[H23 ? 2 : 1][H23 ? PHN : 1];  // H23: hat values of dimensions 2, 3 (registers)
    T h0[H0 ? 3 : 1];                      // H0: level-0 hat values of dimensions 2, 3, 4 (registers)
    uint32_t K[D];
    double res;  // the query's sum over the blocks: fp64 also for fp32 storage (reading G13: a long
                 // sequential fp32 accumulation would lose ~sqrt(#blocks) ulps of fp32)
    uint32_t b;  // running subspace base (elements), warp-uniform
  };

  // shared-memory hat value (GO: 1)
  static __device__ __forceinline__ T phs_at(const T* phs, int row) { return GO ? T(1) : phs[row * NT]; }

  static constexpr uint32_t cnt(int R, int NI) {  // subspaces per block = C(R+NI-1, NI-1)
    uint32_t c = 1;
    for (int k = 1; k <= NI - 1; ++k) c = c * (uint32_t)(R + k) / (uint32_t)k;
    return c;
  }

  // ---------------------------------------------------------------- leaf block
  // Group J, R = J - sigma: every shift below is a compile-time constant.
  template <int J, int R>
  static __device__ __forceinline__ void block(Ctx& c, uint32_t P, T prod) {
    constexpr int NI = I;
    if constexpr ((R < RMIN && !KN::RMIN_NODES_ONLY) || R > RMAX) {  // another launch evaluates this block
      c.b += cnt(R, NI) << J;
      return;
    } else {
      block_eval<J, R>(c, P, prod);
    }
  }
  // number of subspaces of the sub-trie of dimensions t..0 with level sum B (l_0 implied): C(B+t, t)
  template <int t>
  static __device__ __forceinline__ uint32_t nsub(int B) {
    uint32_t r = 0;
#pragma unroll
    for (int b = 0; b < NM; ++b)
      if (b == B) r = binom_c(b + t, t);
    return r;
  }
  static constexpr uint32_t binom_c(int a, int b) {
    uint32_t c = 1;
    for (int k = 1; k <= b; ++k) c = c * (uint32_t)(a - b + k) / (uint32_t)k;
    return c;
  }

  template <int J, int R>
  static __device__ __forceinline__ void block_eval(Ctx& c, uint32_t P, T prod) {
    constexpr int NI = I;
    constexpr int SG = J - R;  // sigma = sum of the outer levels
    // per-lane block base &alpha[b + P] (P = the outer digits, all below bit SG)
    const T* base = c.alpha + c.b + P;
    uint32_t k0, k1, k2, k3;  // opaque copies: keep the per-block cell work inside the trie
    asm volatile("mov.b32 %0, %1;" : "=r"(k0) : "r"(c.K[0]));
    asm volatile("mov.b32 %0, %1;" : "=r"(k1) : "r"(c.K[NI > 1 ? 1 : 0]));
    asm volatile("mov.b32 %0, %1;" : "=r"(k2) : "r"(c.K[NI > 2 ? 2 : 0]));
    asm volatile("mov.b32 %0, %1;" : "=r"(k3) : "r"(c.K[NI > 3 ? 3 : 0]));
    // C'[s] = (k_0(R-s) << (s+SG)) | (k_1 digits at level s, shifted by SG);
    // bits below SG are garbage and cleared by every row mask.
    const uint32_t K0J = k0 >> (NM - 1 - J);
    uint32_t Cs[R + 1];
#pragma unroll
    for (int s = 0; s <= R; ++s) {
      if constexpr (CST) {
        Cs[s] = c.ct[CST ? s + SG : 0];
      } else {
        const uint32_t hi = K0J & ~((1u << (s + SG)) - 1u);
        const uint32_t lo = (NI > 1) ? (k1 >> (NM - 1 - s - SG)) : 0u;
        Cs[s] = hi | lo;
      }
    }
    // hat values of dimensions 2, 3 for levels 0..R, from shared memory
    T ph2[R + 1], ph3[LZ3 ? 1 : R + 1];
#pragma unroll
    for (int l = 0; l <= R; ++l) {
      if constexpr (H23) {
        ph2[l] = c.ph23[0][H23 ? l : 0];
        if constexpr (!LZ3) ph3[l] = c.ph23[H23 ? 1 : 0][H23 ? l : 0];
      } else {
        ph2[l] = (NI >= 3) ? ((H0 && l == 0) ? c.h0[0] : phs_at(c.phs, 0 * PHB + l)) : T(1);
        if constexpr (!LZ3)
          ph3[l] = (NI >= 4) ? ((H0 && l == 0) ? c.h0[H0 ? 1 : 0] : phs_at(c.phs, 1 * PHB + l)) : T(1);
      }
    }
    // INNER = 5: hat values of dimension 4 for levels 0..R, from shared memory
    T ph4[NI >= 5 ? R + 1 : 1];
    uint32_t k4 = 0;
    if constexpr (NI >= 5) {
#pragma unroll
      for (int l = 0; l <= R; ++l) ph4[l] = (H0 && l == 0) ? c.h0[H0 ? 2 : 0] : phs_at(c.phs, 2 * PHB + l);
      asm volatile("mov.b32 %0, %1;" : "=r"(k4) : "r"(c.K[NI > 4 ? 4 : 0]));
    }
    T acc = T(0);
    constexpr int R4 = (NI >= 5) ? R : 0;
    int cidx = 0;  // compile-time after unrolling: rank of the term inside the block
#pragma unroll
    for (int l4 = 0; l4 <= R4; ++l4) {
      // k_4(l4) << SG (INNER = 5); the dimensions <= 3 sit above bit SG4
      const int SG4 = SG + l4;
      const uint32_t X4 = (NI >= 5) ? ((k4 >> (NM - 1 - l4 - SG)) & ~((1u << SG) - 1u)) : 0u;
      const int R3 = (NI >= 4) ? R - l4 : 0;
      T acc4 = T(0);
#pragma unroll
      for (int l3 = 0; l3 <= R3; ++l3) {
        // k_3(l3) << SG4
        const uint32_t X3 = (NI >= 4) ? (((k3 >> (NM - 1 - l3 - SG4)) & ~((1u << SG4) - 1u)) | X4) : X4;
        const int R2 = (NI >= 3) ? R - l4 - l3 : 0;
        T acc3 = T(0);
#pragma unroll
        for (int l2 = 0; l2 <= R2; ++l2) {
          // X_row = (k_2(l2) << (l3+SG4)) | X3
          uint32_t Xr = (NI >= 3) ? (((k2 >> (NM - 1 - l2 - l3 - SG4)) & ~((1u << (l3 + SG4)) - 1u)) | X3) : X3;
          asm("mov.b32 %0, %0;" : "+r"(Xr));
          const uint32_t M = 0xffffffffu << (l2 + l3 + SG4);
          const int R1 = (NI >= 2) ? R - l4 - l3 - l2 : 0;
          T acc2 = T(0);
#pragma unroll
          for (int l1 = 0; l1 <= R1; ++l1) {
            const int s = l1 + l2 + l3 + l4;
            const int l0 = R - s;
            uint32_t V;  // index1 - P = (C'[s] & M_row) | X_row: one LOP3
            asm("lop3.b32 %0, %1, %2, %3, 0xEA;" : "=r"(V) : "r"(Cs[s]), "r"(M), "r"(Xr));
            const T* p;  // &alpha[b + P + V] (one LEA pair); the term's c * 2^J is the load's immediate
            asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(p) : "r"(V), "n"((int)sizeof(T)), "l"(base));
            const T a = __ldg(p + ((uint32_t)cidx << J));
            if constexpr (D01) {
              const int r = R - l2 - l3 - l4;
              acc2 = fma(a, c.d01[D01 ? r * (r + 1) / 2 + l1 : 0], acc2);
            } else if (NI >= 2) {
              acc2 = fma(a * c.ph[0][D01 ? 0 : l0], c.ph[NI > 1 ? 1 : 0][D01 ? 0 : l1], acc2);
            } else {
              acc2 = fma(a, c.ph[0][D01 ? 0 : l0], acc2);
            }
            ++cidx;
          }
          acc3 = (NI >= 3) ? fma(acc2, ph2[l2], acc3) : acc2;
        }
        if constexpr (NI >= 4) {
          const T h3 = LZ3 ? phs_at(c.phs, 1 * PHB + l3) : ph3[LZ3 ? 0 : l3];
          acc4 = fma(acc3, h3, acc4);
        } else {
          acc4 = acc3;
        }
      }
      acc = (NI >= 5) ? fma(acc4, ph4[NI >= 5 ? l4 : 0], acc) : acc4;
    }
    c.res = fma((double)acc, (double)prod, c.res);
    c.b += cnt(R, NI) << J;
  }

  // ------------------------------------------------------- outer trie levels
  // node<J, t>: the sub-trie of dimensions t .. 0 whose levels sum to B
  // (l_0 implied), under the outer digits P (dimensions > t, all below bit
  // J - B) and their hat product `prod`.  Dimension I (the innermost outer
  // dimension) is emitted as straight-line code for B <= kFull, and its last
  // kTail + 1 blocks (the small ones, R <= kTail: 1 + 4 + 10 + 20 terms) are
  // merged into one basic block (kTail = 3 measured 2.8% faster than 2), so
  // that each basic block keeps more surplus loads in flight (v2 issued one
  // small block at a time and was latency-bound, profiles/r01_v2_*).
  // Straight-line sub-tries of higher dimensions thrash the instruction cache
  // (23.7% no_instruction stalls at 70 terms, profiles/r01_v3_variants.txt):
  // only budget-0 sub-tries of dimensions > I are straight-line.

  // hat value from u = 2^l x - k(l) in [0, 1] (reading G7): 2 min(u, 1-u) = 2u if 2u < 1, else 2 - 2u -- exact
  // (2u is exact, 2 - 2u by Sterbenz).  Queries with a coordinate outside [0, 1] never use these values: their
  // result is set to 0 (f_s = 0 outside the domain, reading G8), so no clamp is needed here.
  static __device__ __forceinline__ T hat_u(T u) {
    if constexpr (GO) return T(1);
    const T t = u + u;
    return t < T(1) ? t : T(2) - t;
  }
  // u_{l+1} = frac(2 u_l), exact for u in [0, 1]; u = 1 (x = 1, the clamped last cell) stays 1 (hat 0)
  static __device__ __forceinline__ T dbl_u(T u) {
    u = u + u;
    return u >= T(1) ? u - T(1) : u;
  }

  // dimension I at compile-time budget B: levels l = L .. B unrolled into one basic block
  template <int J, int B, int L>
  static __device__ __forceinline__ void inner_unrolled(Ctx& c, uint32_t P, T prod, T u) {
    if constexpr (L <= B) {
      constexpr int SG = J - B;
      const T ph = IDBL ? hat_u(u) : phs_at(c.phs, SM_IN + L);
      const uint32_t kt = c.K[I] >> (NM - 1 - L);
      block<J, B - L>(c, P | (kt << SG), prod * ph);
      inner_unrolled<J, B, L + 1>(c, P, prod, IDBL ? dbl_u(u) : u);
    }
  }

  // sub-trie of dimensions t .. 0 at compile-time budget B, straight-line
  template <int J, int t, int B>
  static __device__ __forceinline__ void flat(Ctx& c, uint32_t P, T prod) {
    if constexpr (S0 && B == 0 && t >= I) {
      // every level of dimensions t..0 is 0: the single subspace of this
      // sub-trie, cell 0 in each of those dimensions (digits of length 0)
      const T a = __ldg(c.alpha + c.b + P);
      c.res = fma((double)a, (double)(prod * c.s0[(t - I) * NT]), c.res);
      c.b += 1u << J;
    } else if constexpr (t < I) {
      block<J, B>(c, P, prod);
    } else if constexpr (t == I) {
      inner_unrolled<J, B, 0>(c, P, prod, IDBL ? c.xs[0] : T(0));
    } else {
      static_assert(B == 0, "only budget-0 sub-tries above dimension I are straight-line");
      // level 0 of dimension t: digit of length 0, hat phi_0(x_t)
      flat<J, t - 1, 0>(c, P, prod * hat_u(c.xs[xrow(t) * NT]));
    }
  }

#define SG_TRIE_FULL(k) \
  case k:               \
    if constexpr (k <= kFull && k <= J) flat<J, I, (k <= kFull && k <= J ? k : 0)>(c, P, prod); \
    break;
  // dimension I at a small run-time budget: the compile-time straight-line sub-tries
  template <int J>
  static __device__ __forceinline__ void inner_dispatch(Ctx& c, int B, uint32_t P, T prod) {
    switch (B) {
      SG_TRIE_FULL(0) SG_TRIE_FULL(1) SG_TRIE_FULL(2) SG_TRIE_FULL(3)
      SG_TRIE_FULL(4) SG_TRIE_FULL(5) SG_TRIE_FULL(6) SG_TRIE_FULL(7)
      default: break;
    }
  }
#undef SG_TRIE_FULL

  // tail of dimension I at run-time budget B: the blocks R = RT .. 0
  // (l_I = B - R), merged into one basic block
  template <int J, int RT>
  static __device__ __forceinline__ void inner_tail(Ctx& c, int B, uint32_t P, T prod, T u) {
    if constexpr (RT >= 0) {
      const int lt = B - RT;
      const T ph = IDBL ? hat_u(u) : phs_at(c.phs, SM_IN + lt);
      const uint32_t kt = c.K[I] >> (NM - 1 - lt);
      block<J, RT>(c, P | (kt << (J - B)), prod * ph);
      inner_tail<J, RT - 1>(c, B, P, prod, IDBL ? dbl_u(u) : u);
    }
  }

#define SG_TRIE_CASE(r) \
  case r:               \
    if constexpr (r <= J) block<J, (r <= J ? r : 0)>(c, P, prod); \
    break;
  template <int J>
  static __device__ __forceinline__ void leaf(Ctx& c, int R, uint32_t P, T prod) {
    switch (R) {
      SG_TRIE_CASE(0) SG_TRIE_CASE(1) SG_TRIE_CASE(2) SG_TRIE_CASE(3)
      SG_TRIE_CASE(4) SG_TRIE_CASE(5) SG_TRIE_CASE(6) SG_TRIE_CASE(7)
      SG_TRIE_CASE(8) SG_TRIE_CASE(9) SG_TRIE_CASE(10) SG_TRIE_CASE(11)
      SG_TRIE_CASE(12) SG_TRIE_CASE(13) SG_TRIE_CASE(14) SG_TRIE_CASE(15)
      default: break;
    }
  }
#undef SG_TRIE_CASE

  // S0, budget 1 at dimension t > I: the t + 1 subspaces with one level-1
  // dimension u (u = 0..t, in the bijection order, Alg. 3: u = 0 first) and
  // every other level of dimensions t..0 zero are consecutive; dimension u's
  // one-bit digit k_u(1) sits just above the outer digits P (bit J - 1).
  // Their sum sum_u alpha_u phi_1(x_u) prod_{v<=t, v!=u} phi_0(x_v) is
  // S0[t] * sum_u alpha_u rho_u (Alg. 7's product of hat values).
  template <int J, int t>
  static __device__ __forceinline__ void budget1(Ctx& c, uint32_t P, T prod) {
    const T* base = c.alpha + c.b + P;
    T acc = T(0);
#pragma unroll
    for (int u = 0; u <= t; ++u) {
      const T r = c.rho[u * NT];
      const uint32_t k1 = (uint32_t)__double2hiint((double)r) >> 31;  // k_u(1), the sign bit
      const T a = __ldg(base + ((k1 << (J - 1)) + ((uint32_t)u << J)));
      acc = fma(a, fabs(r), acc);
    }
    c.res = fma((double)acc, (double)(prod * c.s0[(t - I) * NT]), c.res);
    c.b += (uint32_t)(t + 1) << J;
  }

  // node at dimension t >= I with run-time budget B (levels of dimensions
  // t..0 sum to B): a run-time loop over l_t, each child inlined once
  template <int J, int t>
  static __device__ __forceinline__ void node(Ctx& c, int B, uint32_t P, T prod) {
    if constexpr (RMIN > 0) {
      if (B < RMIN) {  // every block of this sub-trie has R <= B < RMIN: another launch's
        c.b += nsub<t>(B) << J;
        return;
      }
    }
    if constexpr (S0 && t > I && J >= 1 && NM >= 2) {
      if (B == 1) {
        budget1<J, t>(c, P, prod);
        return;
      }
    }
    const int SG = J - B;  // shift of dimension t's digit
    if constexpr (t == I) {
      if (B <= kFull) {
        inner_dispatch<J>(c, B, P, prod);
        return;
      }
      T u = IDBL ? c.xs[0] : T(0);  // IDBL: u = 2^lt x_I - k_I(lt) along the level loop
      for (int lt = 0; lt < B - kTail; ++lt) {
        const T ph = IDBL ? hat_u(u) : phs_at(c.phs, SM_IN + lt);
        const uint32_t kt = c.K[I] >> (NM - 1 - lt);
        leaf<J>(c, B - lt, P | (kt << SG), prod * ph);
        if constexpr (IDBL) u = dbl_u(u);
      }
      inner_tail<J, kTail>(c, B, P, prod, u);
    } else {
      if (B == 0) {
        flat<J, t, 0>(c, P, prod);
        return;
      }
      T u = c.xs[xrow(t) * NT];
      for (int lt = 0; lt <= B; ++lt) {
        if constexpr (KN::SYNC == t) __syncthreads();
        const uint32_t kt = c.K[t] >> (NM - 1 - lt);
        node<J, t - 1>(c, B - lt, P | (kt << SG), prod * hat_u(u));
        u = dbl_u(u);
      }
    }
  }

  template <int J, int J1>
  static __device__ __forceinline__ void groups(Ctx& c, int n) {
    if constexpr (J <= J1 && J < NM) {
      if (J < n) {
        if constexpr (CST) {
          const uint32_t K0J = c.K[0] >> (NM - 1 - J);
#pragma unroll
          for (int u = 0; u <= J; ++u)
            c.ct[CST ? u : 0] = (K0J & ~((1u << u) - 1u)) | ((I > 1) ? (c.K[I > 1 ? 1 : 0] >> (NM - 1 - u)) : 0u);
        }
        if constexpr (O == 0) block<J, J>(c, 0u, T(1));  // no outer dimensions: one block per group
        else node<J, D - 1>(c, J, 0u, T(1));
        groups<J + 1, J1>(c, n);
      }
    }
  }
};


// One launch evaluates the level groups J0..J1 (compile time) for every
// query; launches of consecutive ranges accumulate into y (accumulate = 0 for
// the first range).  b0 = index3(J0), the offset of group J0.
// One query per thread (q = its position in the order perm), shared-memory column tid.
template <typename T, int D, int NM, int NT, int J0, int J1, class KN>
__device__ __forceinline__ void eval_query(const T* __restrict__ alpha, const T* __restrict__ x,
                                           const uint32_t* __restrict__ perm, uint32_t m, int n, uint32_t b0,
                                           int accumulate, T* __restrict__ y, T* sm, int tid, uint32_t q) {
  using TR = Trie<T, D, NM, NT, KN>;
  constexpr int I = TR::I;
  const bool active = q < m;
  const uint32_t src = active ? (perm ? perm[q] : q) : 0u;

  typename TR::Ctx c;
  c.alpha = alpha;
  c.phs = sm + tid;
  c.xs = sm + (TR::SM_IN + TR::SM_PH) * NT + tid;
  c.s0 = sm + (TR::SM_IN + TR::SM_PH + TR::SM_X) * NT + tid;
  c.rho = sm + (TR::SM_IN + TR::SM_PH + TR::SM_X + TR::SM_S0) * NT + tid;
  T p0 = T(1);  // S0: running product of the level-0 hat values
  // ---- a2: finest cells of every dimension; hat values of every level of
  // dimensions 0..I (registers for 0, 1; shared memory for 2, 3, I)
  bool bad = false, outside = false;
  const T fine = (T)(1u << (NM - 1));
  T h01[2][TR::PHN];  // D01: hat values of dimensions 0, 1 before their pairwise products
#pragma unroll
  for (int t = 0; t < D; ++t) {
    const T xt = active ? x[(size_t)src * D + t] : T(0.5);
    bad |= isnan(xt);
    outside |= !(xt >= T(0) && xt <= T(1));
    T kf = floor(xt * fine);
    kf = kf > T(0) ? kf : T(0);
    kf = kf < fine - T(1) ? kf : fine - T(1);
    c.K[t] = (uint32_t)kf;
    if constexpr (TR::SM_S0 > 0) {
      uint32_t cell0;
      p0 *= hat_cell<T>(xt, 0, cell0);
      if (t >= I) sm[(TR::SM_IN + TR::SM_PH + TR::SM_X + (t - I)) * NT + tid] = p0;
    }
    if constexpr (TR::SM_RHO > 0) {
      uint32_t c0, c1;
      const T f0 = hat_cell<T>(xt, 0, c0), f1 = hat_cell<T>(xt, 1, c1);
      const double r = f0 > T(0) ? (double)(f1 / f0) : 0.0;
      const long long bits = __double_as_longlong(r) | ((long long)(c1 & 1u) << 63);
      sm[(TR::SM_IN + TR::SM_PH + TR::SM_X + TR::SM_S0 + t) * NT + tid] = (T)__longlong_as_double(bits);
    }
    if (t < I || (t == I && !TR::IDBL)) {
#pragma unroll
      for (int l = 0; l < NM; ++l) {
        uint32_t cell;
        const T h = KN::GO ? T(1) : hat_cell<T>(xt, l, cell);
        if (t < 2) {
          if (l < TR::PHN) {
            if constexpr (TR::D01) h01[t < 2 ? t : 0][l < TR::PHN ? l : 0] = h;
            else c.ph[t < 2 ? t : 0][l < TR::PHN ? l : 0] = h;
          }
        } else if (TR::H23 && t < 4 && l < TR::PHN) {
          c.ph23[TR::H23 ? t - 2 : 0][TR::H23 && l < TR::PHN ? l : 0] = h;
        }
        else if (t < I) {
          if (l < TR::PHB) sm[((t - 2) * TR::PHB + (l < TR::PHB ? l : 0)) * NT + tid] = h;
          if (TR::H0 && l == 0) c.h0[TR::H0 ? (t < 5 ? t - 2 : 0) : 0] = h;
        }
        else sm[(TR::SM_IN + l) * NT + tid] = h;
      }
    } else {
      sm[(TR::SM_IN + TR::SM_PH + TR::xrow(t)) * NT + tid] = xt;
    }
  }
  if constexpr (TR::D01) {
#pragma unroll
    for (int r = 0; r < TR::PHN; ++r)
#pragma unroll
      for (int l1 = 0; l1 <= r; ++l1) c.d01[r * (r + 1) / 2 + l1] = h01[0][r - l1] * h01[1][l1];
  }
  // (no barrier: every lane reads only its own shared-memory column)
  c.res = 0.0;
  c.b = b0;
  TR::template groups<J0, J1>(c, n);
  if (active) {
    double r = c.res;
    if (accumulate) r += (double)y[src];
    y[src] = bad ? T(NAN) : (outside ? T(0) : (T)r);
  }
}

template <typename T, int D, int NM, int NT, int MINB, int J0, int J1, class KN>
__global__ void __launch_bounds__(NT, MINB)
    k_eval_trie(const T* __restrict__ alpha, const T* __restrict__ x, const uint32_t* __restrict__ perm, uint32_t m,
                int n, uint32_t b0, int accumulate, T* __restrict__ y) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  eval_query<T, D, NM, NT, J0, J1, KN>(alpha, x, perm, m, n, b0, accumulate, y, reinterpret_cast<T*>(smem_raw),
                                       threadIdx.x, blockIdx.x * NT + threadIdx.x);
}

template <typename T, int D, int NM, int NT, int MINB, int J0, int J1, class KN = Knobs>
sg_status launch_range(const Layout& L, const T* alpha, const T* x, const uint32_t* perm, uint64_t m, T* y,
                       cudaStream_t s) {
  if (J0 >= L.n) return SG_OK;
  using TR = Trie<T, D, NM, NT, KN>;
  auto kern = k_eval_trie<T, D, NM, NT, MINB, J0, J1, KN>;
  const size_t smem = TR::smem_bytes;
  // shared memory only for the per-lane tables: the rest of the 256 KB stays L1
  // for the surplus gathers
  const int pct = (int)((smem * MINB * 100 + 227 * 1024 - 1) / (227 * 1024)) + 1;
  static std::atomic<uint64_t> attr_done{0};
  const sg_status st = set_smem_attr(kern, attr_done, smem, pct, "cudaFuncSetAttribute(k_eval_trie)");
  if (st != SG_OK) return st;
  const unsigned blocks = (unsigned)((m + NT - 1) / NT);
  // the first launch of a call (group 0, all budgets) writes y, every later one accumulates
  const int accumulate = (J0 > 0 || KN::RMIN > 0) ? 1 : 0;
  kern<<<blocks, NT, smem, s>>>(alpha, x, perm, (uint32_t)m, L.n, (uint32_t)L.off[J0], accumulate, y);
  return launched("k_eval_trie", (const void*)kern);
}

}  // namespace trie
}  // namespace sg
