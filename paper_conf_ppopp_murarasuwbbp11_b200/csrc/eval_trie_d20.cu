// eval_trie_d20.cu -- instantiations of the v2 evaluation kernel (eval_trie.cuh) for d = 20, n <= 6 (cfg5).
// One launch per level-group range; consecutive launches accumulate into y.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_trie.cuh"

namespace sg {

sg_status trie_d20n6(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 20, 6, 128, 3, 0, 5, trie::KnobsS0>(L, a, x, p, m, y, s);
  return st;
}

}  // namespace sg
