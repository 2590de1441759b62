// BSY9: the v9.1 product (barrier per level step of dimension 9) with 512-thread small-block CTAs (1 per SM)
#include "exp_sync.cuh"
namespace sg {
sg_status exp_BSY9(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                   cudaStream_t s) {
  using namespace v9;
  return run<KLowS<6, 9>, KLowS<4, 9>, KHighS<4, 9>, 512, 1, 128, 3>(L, a, x, p, m, y, s);
}
}  // namespace sg
