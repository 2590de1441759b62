// eval_trie_d10a.cu -- instantiations of the evaluation kernel (eval_trie.cuh) for d = 10, n <= 11 (cfg3),
// groups 0..8.  One launch per (level-group range, block-budget range); consecutive launches accumulate
// into y.  Groups >= 7 are split by budget: the small-block launch evaluates the sub-tries of dimensions
// 0..4 whose level sum is <= 4 as blocks of 5 inner dimensions (INNER = 5: C(R+4, 4) consecutive
// subspaces per block) with the register hat tables of dimensions 0, 1 only up to level 4, at 16
// warps/SM (128 registers); the large-block launch (blocks over dimensions 0..3, 12 warps/SM) prunes
// exactly those sub-tries.  Groups 0-6 run as small blocks (R <= 6) at 16 warps/SM.  Measured +8% (split
// at 4 dimensions) and +3% more (5 inner dimensions for the small blocks) over one launch per group at 12
// warps/SM (profiles/r02_split.txt).  v9: the small-block launches run as 256-thread CTAs (2 per SM:
// 8 warps of neighbouring queries share the SM's L1) with hat rows of dimensions 2..4 only up to level
// RMAX (18 KB less shared memory per 128 queries, so more L1) and the level-0 hats of dimensions 2..4 in
// registers: +4.2%, +2.5% and +1.2%; a CTA barrier per level step of dimension 9 keeps the warps of a CTA
// in step (+1.3%) (profiles/r02_v9.txt).  Split across files only so that nvcc
// compiles them in parallel.
#include "eval_trie.cuh"

namespace sg {

namespace d10 {
// small blocks: sub-tries of dimensions 0..4 (INNER = 5) with level sum <= RL
template <int RL>
struct KLow : trie::Knobs {
  static constexpr int RMAX = RL;
  static constexpr int INNER = 5;
  static constexpr bool H0 = true;  // level-0 hats of dimensions 2..4 in registers (+1.2%, profiles/r02_v9.txt)
  static constexpr int SYNC = 9;    // CTA barrier per level step of dimension 9 (+1.3%, profiles/r02_v9.txt)
};
// large blocks: blocks over dimensions 0..3 of every dimension-4 node with budget > RL (exactly the
// complement: the nodes of budget <= RL are the small-block launch's blocks)
template <int RL>
struct KHigh : trie::Knobs {
  static constexpr int RMIN = RL + 1;
  static constexpr bool RMIN_NODES_ONLY = true;
  static constexpr int SYNC = 9;
  static constexpr bool IDBL = true;  // dimension-4 hats by doubling: 10 smem rows less, more L1 (+1.6%, r02_v9.txt)
};
}  // namespace d10

sg_status trie_d10n11_a(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                        cudaStream_t s) {
  using namespace d10;
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 256, 2, 0, 6, KLow<6>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 256, 2, 7, 7, KLow<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 7, 7, KHigh<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 256, 2, 8, 8, KLow<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 8, 8, KHigh<4>>(L, a, x, p, m, y, s);
  return st;
}

}  // namespace sg
