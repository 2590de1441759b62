// cfg4 (fp32 d = 3, n <= 14) and cfg2/cfg2' (d = 5) with larger CTAs (8 / 16 / 12 warps sharing one L1)
#include "../eval_trie.cuh"

namespace sg {
template <int NT, int MB>
static sg_status d3f(const Layout& L, const float* a, const float* x, const uint32_t* p, uint64_t m, float* y,
                     cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, NT, MB, 0, 7>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, NT, MB, 8, 9>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, NT, MB, 10, 11>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<float, 3, 14, NT, MB, 12, 13>(L, a, x, p, m, y, s);
  return st;
}
sg_status exp_D3T256(const Layout& L, const float* a, const float* x, const uint32_t* p, uint64_t m, float* y,
                     cudaStream_t s) {
  return d3f<256, 2>(L, a, x, p, m, y, s);
}
sg_status exp_D3T512(const Layout& L, const float* a, const float* x, const uint32_t* p, uint64_t m, float* y,
                     cudaStream_t s) {
  return d3f<512, 1>(L, a, x, p, m, y, s);
}
sg_status exp_D5T384(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                     cudaStream_t s) {
  sg_status st = SG_OK;
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 384, 1, 0, 5>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 384, 1, 6, 6>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 384, 1, 7, 7>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 384, 1, 8, 8>(L, a, x, p, m, y, s);
  if (st == SG_OK) st = trie::launch_range<double, 5, 10, 384, 1, 9, 9>(L, a, x, p, m, y, s);
  return st;
}
}  // namespace sg
