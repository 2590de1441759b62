// LSY1 / LSY2: the v9.1 product with the large-block launches as 384 x 1 / 192 x 2 CTAs (12 warps/SM in
// one / two barrier-synchronised CTAs)
#include "exp_sync.cuh"
namespace sg {
sg_status exp_LSY1(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                   cudaStream_t s) {
  using namespace v9;
  return run<KLowS<6, 9>, KLowS<4, 9>, KHighS<4, 9>, 256, 2, 384, 1>(L, a, x, p, m, y, s);
}
sg_status exp_LSY2(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                   cudaStream_t s) {
  using namespace v9;
  return run<KLowS<6, 9>, KLowS<4, 9>, KHighS<4, 9>, 256, 2, 192, 2>(L, a, x, p, m, y, s);
}
}  // namespace sg
