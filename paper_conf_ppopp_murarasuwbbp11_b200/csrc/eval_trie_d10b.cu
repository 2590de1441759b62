// eval_trie_d10b.cu -- instantiations of the evaluation kernel (eval_trie.cuh) for d = 10, n <= 11 (cfg3),
// groups 9..10, split by block budget as in eval_trie_d10a.cu.  Split across files only so that nvcc
// compiles them in parallel.
#include "eval_trie.cuh"

namespace sg {

namespace d10b {
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
}  // namespace d10b

sg_status trie_d10n11_b(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                        cudaStream_t s) {
  using namespace d10b;
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 256, 2, 9, 9, KLow<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 9, 9, KHigh<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 256, 2, 10, 10, KLow<4>>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 10, 10, KHigh<4>>(L, a, x, p, m, y, s);
  return st;
}

}  // namespace sg
