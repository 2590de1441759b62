// LH4 / LH42: the v9.1 product with the large-block launches at 16 warps/SM (128 registers): 128 x 4 / 256 x 2
#include "exp_sync.cuh"
namespace sg {
sg_status exp_LH4(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                  cudaStream_t s) {
  using namespace v9;
  return run<KLowS<6, 9>, KLowS<4, 9>, KHighS<4, 9>, 256, 2, 128, 4>(L, a, x, p, m, y, s);
}
sg_status exp_LH42(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                   cudaStream_t s) {
  using namespace v9;
  return run<KLowS<6, 9>, KLowS<4, 9>, KHighS<4, 9>, 256, 2, 256, 2>(L, a, x, p, m, y, s);
}
}  // namespace sg
