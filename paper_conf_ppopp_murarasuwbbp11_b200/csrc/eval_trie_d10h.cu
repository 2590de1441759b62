// eval_trie_d10h.cu -- experiment variant of the d = 10, n <= 11 evaluation kernel: hat values of dimension 4
// by exact doubling along its loop instead of a shared-memory table (eval_trie.cuh H4; SG_TRIE_VAR=H).
#include "eval_trie.cuh"

namespace sg {

sg_status trie_d10n11_h4(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                         cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 0, 6, 0, false, 3, false, 0, 4, 0, true>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 7, 7, 0, false, 3, false, 0, 4, 0, true>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 8, 8, 0, false, 3, false, 0, 4, 0, true>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 9, 9, 0, false, 3, false, 0, 4, 0, true>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 10, 10, 0, false, 3, false, 0, 4, 0, true>(L, a, x, p, m, y, s);
  return st;
}

}  // namespace sg
