// eval_trie_d10x.cu -- experiment variants of the d = 10, n <= 11 evaluation kernel (groups 9..10) with an
// L1 cache-eviction hint on the surplus gathers (eval_trie.cuh ld_surplus; selected by SG_TRIE_VAR).
#include "eval_trie.cuh"

namespace sg {

template <int CH>
static sg_status d10b_ch(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                         cudaStream_t s) {
  sg_status st = trie::launch_range<double, 10, 11, 128, 3, 9, 9, 0, false, 3, false, 0, 4, CH>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, 128, 3, 10, 10, 0, false, 3, false, 0, 4, CH>(L, a, x, p, m, y, s);
  return st;
}

sg_status trie_d10n11_b_hint(int ch, const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m,
                             double* y, cudaStream_t s) {
  switch (ch) {
    case 1: return d10b_ch<1>(L, a, x, p, m, y, s);
    case 2: return d10b_ch<2>(L, a, x, p, m, y, s);
    default: return d10b_ch<3>(L, a, x, p, m, y, s);
  }
}

}  // namespace sg
