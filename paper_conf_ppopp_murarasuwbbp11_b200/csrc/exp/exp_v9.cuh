// exp_v9.cuh -- r02 v9 experiment variants of the cfg3 evaluation (experiment builds only): the product's
// launch structure (eval_trie_d10a/b.cu) with knob and CTA-shape variants; one variant per .cu file so that
// nvcc compiles them in parallel.
#pragma once
#include <type_traits>

#include "../eval_trie.cuh"
#include "exp_pw.cuh"

namespace sg {
namespace v9 {
template <int RL>
struct KHighN : trie::Knobs {
  static constexpr int RMIN = RL + 1;
  static constexpr bool RMIN_NODES_ONLY = true;
};
template <int RL>
struct KHighGO : KHighN<RL> {
  static constexpr bool GO = true;
};
template <int RL, bool TA, bool HZ, bool ID = false, bool G = false>
struct KLow9 : trie::Knobs {
  static constexpr int RMAX = RL;
  static constexpr int INNER = 5;
  static constexpr bool TAB_ALL = TA;
  static constexpr bool H0 = HZ;
  static constexpr bool IDBL = ID;
  static constexpr bool GO = G;
};
template <class KL06, class KL, class KH, int NTL, int MBL, int NTH, int MBH, bool PW = false>
sg_status run(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
              cudaStream_t s) {
  sg_status st = SG_OK;
  if constexpr (PW) {
    if (st == SG_OK) st = pw::launch_range<double, 10, 11, NTL, MBL, 0, 6, KL06>(L, a, x, p, m, y, s);
  } else {
    if (st == SG_OK) st = trie::launch_range<double, 10, 11, NTL, MBL, 0, 6, KL06>(L, a, x, p, m, y, s);
  }
#define SG_R(J)                                                                                          \
  if constexpr (PW) {                                                                                    \
    if (st == SG_OK) st = pw::launch_range<double, 10, 11, NTL, MBL, J, J, KL>(L, a, x, p, m, y, s);     \
    if (st == SG_OK) st = pw::launch_range<double, 10, 11, NTH, MBH, J, J, KH>(L, a, x, p, m, y, s);     \
  } else {                                                                                               \
    if (st == SG_OK) st = trie::launch_range<double, 10, 11, NTL, MBL, J, J, KL>(L, a, x, p, m, y, s);   \
    if (st == SG_OK) st = trie::launch_range<double, 10, 11, NTH, MBH, J, J, KH>(L, a, x, p, m, y, s);   \
  }
  SG_R(7) SG_R(8) SG_R(9) SG_R(10)
#undef SG_R
  return st;
}
}  // namespace v9
}  // namespace sg

#define SG_V9(name, HZ, ID, G, NTL, MBL, NTH, MBH, ...)                                                              \
  namespace sg {                                                                                              \
  sg_status name(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,   \
                 cudaStream_t s) {                                                                            \
    using namespace v9;                                                                                       \
    using KH = typename std::conditional<G, KHighGO<4>, KHighN<4>>::type;                                     \
    return run<KLow9<6, false, HZ, ID, G>, KLow9<4, false, HZ, ID, G>, KH, NTL, MBL, NTH, MBH, ##__VA_ARGS__>(L, a, x, p, m, y, s); \
  }                                                                                                           \
  }
