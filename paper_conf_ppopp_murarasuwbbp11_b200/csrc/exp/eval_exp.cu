// eval_exp.cu -- EXPERIMENT variants of the evaluation kernel, compiled only into libsg_exp.so
// (build.py --exp; never into the product libsg.so).  Selected at run time by SG_EXP_VAR; used by
// scripts/gpu_exp.sh to measure what bounds the product kernel.
#include <stdlib.h>
#include <string.h>

#include "../eval_trie.cuh"

namespace sg {

struct KnobsGO : trie::Knobs {
  static constexpr bool GO = true;
};
struct KnobsLZ3 : trie::Knobs {
  static constexpr bool LZ3 = true;
};

// GO: gather-only (all hat values 1; same addresses, loads and Horner adds), cfg3 shape
template <int MINB, int NT = 128>
static sg_status d10_go(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                        cudaStream_t s) {
  sg_status st = SG_OK;
#define SG_R(J0, J1) \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, NT, MINB, J0, J1, KnobsGO>(L, a, x, p, m, y, s);
  SG_R(0, 6) SG_R(7, 7) SG_R(8, 8) SG_R(9, 9) SG_R(10, 10)
#undef SG_R
  return st;
}

// product kernel at MINB CTAs of NT threads per SM (register cap 65536 / (NT MINB))
template <int MINB, int NT = 128, class KN = trie::Knobs>
static sg_status d10_minb(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                          cudaStream_t s) {
  sg_status st = SG_OK;
#define SG_R(J0, J1) \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, NT, MINB, J0, J1, KN>(L, a, x, p, m, y, s);
  SG_R(0, 6) SG_R(7, 7) SG_R(8, 8) SG_R(9, 9) SG_R(10, 10)
#undef SG_R
  return st;
}

// groups split by block budget: the small blocks (R <= RL) at MINB_LO CTAs/SM with register hat
// tables up to level RL, the large ones (R > RL) at 3 CTAs/SM
template <int RL>
struct KLow : trie::Knobs {
  static constexpr int RMAX = RL;
};
template <int RL>
struct KHigh : trie::Knobs {
  static constexpr int RMIN = RL + 1;
};
template <int RL, int MINB_LO, int MINB_06>
static sg_status d10_split(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                           double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, MINB_06, 0, 6, KLow<6>>(L, a, x, p, m, y, s);
#define SG_R(J)                                                                                          \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, MINB_LO, J, J, KLow<RL>>(L, a, x, p, m, y, s); \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, J, J, KHigh<RL>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}

template <int LO, int HI>
struct KRange : trie::Knobs {
  static constexpr int RMIN = LO;
  static constexpr int RMAX = HI;
};
// three launches per group from 7: R <= A at MINB_A, A < R <= B at 4, R > B at 3; groups 0-6 at 4
template <int A, int B, int MINB_A>
static sg_status d10_split3(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                            double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLow<6>>(L, a, x, p, m, y, s);
#define SG_R(J)                                                                                                \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, MINB_A, J, J, KRange<0, A>>(L, a, x, p, m, y, s);     \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, J, J, KRange<A + 1, B>>(L, a, x, p, m, y, s);      \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, J, J, KRange<B + 1, 64>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}

template <int RL, bool HH, int TL, bool DD = false, bool CT = false>
struct KLowX : trie::Knobs {
  static constexpr int RMAX = RL;
  static constexpr bool H23 = HH;
  static constexpr int TAIL = TL;
  static constexpr bool D01 = DD;
  static constexpr bool CST = CT;
};
template <bool DD, bool CT>
static sg_status d10_splitc(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                            double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLowX<6, false, 3, false, CT>>(L, a, x, p, m, y, s);
#define SG_R(J)                                                                                                        \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, J, J, KLowX<4, false, 3, DD, CT>>(L, a, x, p, m, y, s); \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, J, J, KHigh<4>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}
template <int RL>
static sg_status d10_splitd(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                            double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLowX<6, false, 3, false>>(L, a, x, p, m, y, s);
#define SG_R(J)                                                                                                    \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, J, J, KLowX<RL, false, 3, true>>(L, a, x, p, m, y, s); \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, J, J, KHigh<RL>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}
template <bool HH, int TL>
static sg_status d10_splitx(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                            double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLowX<6, HH, 3>>(L, a, x, p, m, y, s);
#define SG_R(J)                                                                                              \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, J, J, KLowX<4, HH, TL>>(L, a, x, p, m, y, s); \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, J, J, KHigh<4>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}

// cfg5 (d = 20, n = 6, S0 knob): occupancy and block-budget splits
template <int LO, int HI>
struct KS0R : trie::KnobsS0 {
  static constexpr int RMIN = LO;
  static constexpr int RMAX = HI;
};
template <int MINB>
static sg_status d20_minb(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                          cudaStream_t s) {
  return trie::launch_range<double, 20, 6, 128, MINB, 0, 5, trie::KnobsS0>(L, a, x, p, m, y, s);
}
template <int RL, int MINB_LO>
static sg_status d20_split(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                           double* y, cudaStream_t s) {
  sg_status st = trie::launch_range<double, 20, 6, 128, MINB_LO, 0, 5, KS0R<0, RL>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 20, 6, 128, 3, 0, 5, KS0R<RL + 1, 64>>(L, a, x, p, m, y, s);
  return st;
}

template <int RL>
struct KHigh3 : trie::Knobs {
  static constexpr int RMIN = RL + 1;
  static constexpr int INNER = 3;
};
// the large-block launch with blocks over dimensions 0..2 (dimension 3 a trie loop), at MINB_HI CTAs/SM
template <int MINB_HI, bool DD>
static sg_status d10_splith(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                            double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLowX<6, false, 3, false>>(L, a, x, p, m, y, s);
#define SG_R(J)                                                                                                    \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, J, J, KLowX<4, false, 3, DD>>(L, a, x, p, m, y, s); \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, MINB_HI, J, J, KHigh3<4>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}

// INNER = 5 for the small-block launch: blocks = sub-tries of dimensions 0..4 with level sum <= RL;
// the large-block launch (INNER = 4) prunes exactly those sub-tries (node budget at dimension 4 <= RL)
template <int RL>
struct KLow5 : trie::Knobs {
  static constexpr int RMAX = RL;
  static constexpr int INNER = 5;
};
template <int RL>
struct KHighN : trie::Knobs {
  static constexpr int RMIN = RL + 1;
  static constexpr bool RMIN_NODES_ONLY = true;
};
template <int RL, bool I5LOW06>
static sg_status d10_split5(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                            double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if constexpr (I5LOW06) {
    if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLow5<6>>(L, a, x, p, m, y, s);
  } else {
    if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLow<6>>(L, a, x, p, m, y, s);
  }
#define SG_R(J)                                                                                          \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, J, J, KLow5<RL>>(L, a, x, p, m, y, s);  \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, J, J, KHighN<RL>>(L, a, x, p, m, y, s);
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}

// returns true if an experiment variant handled the call
bool exp_dispatch(const Layout& L, const void* alpha, const void* x, const uint32_t* perm, uint64_t m, void* y,
                  sg_dtype dt, cudaStream_t s, sg_status* st) {
  const char* v = getenv("SG_EXP_VAR");
  if (!v || dt != SG_F64) return false;
  if (L.d == 20 && L.n == 6) {
    const double* a = (const double*)alpha;
    if (!strcmp(v, "D20M4")) { *st = d20_minb<4>(L, a, (const double*)x, perm, m, (double*)y, s); return true; }
    if (!strcmp(v, "D20S2")) { *st = d20_split<2, 4>(L, a, (const double*)x, perm, m, (double*)y, s); return true; }
    if (!strcmp(v, "D20S3")) { *st = d20_split<3, 4>(L, a, (const double*)x, perm, m, (double*)y, s); return true; }
    return false;
  }
  if (L.d != 10 || L.n != 11) return false;
  const double* a = (const double*)alpha;
  const double* xx = (const double*)x;
  double* yy = (double*)y;
  if (!strcmp(v, "GO3")) { *st = d10_go<3>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "GO4")) { *st = d10_go<4>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SPLIT4B")) { *st = d10_split<4, 4, 4>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SD4")) { *st = d10_splitd<4>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SC")) { *st = d10_splitc<false, true>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SCD")) { *st = d10_splitc<true, true>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "S5A4")) { *st = d10_split5<4, false>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "S5A5")) { *st = d10_split5<5, false>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "S5B4")) { *st = d10_split5<4, true>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SXT")) { *st = d10_splitx<false, 4>(L, a, xx, perm, m, yy, s); return true; }
  return false;
}

}  // namespace sg
