// eval_trie_d10a.cu -- instantiations of the evaluation kernel (eval_trie.cuh) for d = 10, n <= 11 (cfg3),
// groups 0..8.  One launch per (level-group range, block-budget range); consecutive launches accumulate
// into y.  Groups >= 7 are split by block budget R: the launch of the many small blocks (R <= 4, ~60%
// of the terms) holds the register hat tables of dimensions 0, 1 only up to level 4 and runs 16
// warps/SM (128 registers, no spills); the launch of the large blocks (R >= 5) keeps 12 warps/SM and
// prunes every sub-trie of budget < 5.  Measured +8% over one launch per group at 12 warps
// (profiles/r02_split.txt).  Split across files only so that nvcc compiles them in parallel.
#include "eval_trie.cuh"

namespace sg {

namespace d10 {
template <int RL>
struct KLow : trie::Knobs {
  static constexpr int RMAX = RL;
};
template <int RL>
struct KHigh : trie::Knobs {
  static constexpr int RMIN = RL + 1;
};
}  // namespace d10

sg_status trie_d10n11_a(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                        cudaStream_t s) {
  using namespace d10;
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 0, 6, KLow<6>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 7, 7, KLow<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 7, 7, KHigh<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 4, 8, 8, KLow<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 8, 8, KHigh<4>>(L, a, x, p, m, y, s);
  return st;
}

}  // namespace sg
