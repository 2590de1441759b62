// eval_trie_d10a.cu -- instantiations of the v2 evaluation kernel (eval_trie.cuh) for d = 10, n <= 11 (cfg3), groups 0..8.
// One launch per level-group range; consecutive launches accumulate into y.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_trie.cuh"

namespace sg {

sg_status trie_d10n11_a(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 0, 6>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 7, 7>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 8, 8>(L, a, x, p, m, y, s);
  return st;
}


}  // namespace sg
