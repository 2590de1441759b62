// HH: the v9 product with the level-0 hats of dimensions 2, 3 in registers also in the large-block launch
#include "exp_v9.cuh"
namespace sg {
namespace v9 {
template <int RL>
struct KHighH0 : KHighN<RL> {
  static constexpr bool H0 = true;
};
}  // namespace v9
sg_status exp_HH(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                 cudaStream_t s) {
  using namespace v9;
  return run<KLow9<6, false, true>, KLow9<4, false, true>, KHighH0<4>, 256, 2, 128, 3>(L, a, x, p, m, y, s);
}
// R5: the v9 product split at R <= 5
sg_status exp_R5(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                 cudaStream_t s) {
  using namespace v9;
  return run<KLow9<6, false, true>, KLow9<5, false, true>, KHighN<5>, 256, 2, 128, 3>(L, a, x, p, m, y, s);
}
}  // namespace sg
