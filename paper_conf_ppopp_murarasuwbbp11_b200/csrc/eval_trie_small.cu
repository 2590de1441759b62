// eval_trie_small.cu -- instantiations of the v2 evaluation kernel (eval_trie.cuh) for d = 2, 3, 5.
// One launch per level-group range; consecutive launches accumulate into y.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_trie.cuh"

namespace sg {

sg_status trie_d2n3(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 2, 3, 128, 3, 0, 2>(L, a, x, p, m, y, s);
  return st;
}

sg_status trie_d5n8(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 5, 8, 128, 3, 0, 5>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 8, 128, 3, 6, 6>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 8, 128, 3, 7, 7>(L, a, x, p, m, y, s);
  return st;
}

sg_status trie_d5n10(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 128, 3, 0, 5>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 128, 3, 6, 6>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 128, 3, 7, 7>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 128, 3, 8, 8>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 128, 3, 9, 9>(L, a, x, p, m, y, s);
  return st;
}

sg_status trie_d3n14f(const Layout& L, const float* a, const float* x, const uint32_t* p, uint64_t m, float* y, cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, 128, 4, 0, 7>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, 128, 4, 8, 9>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, 128, 4, 10, 11>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, 128, 4, 12, 13>(L, a, x, p, m, y, s);
  return st;
}

}  // namespace sg
