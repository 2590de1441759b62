// SIDBL: the v9.3 product with the dimension-5 hats of the small-block launches by doubling too (IDBL)
#include "exp_sync.cuh"
namespace sg {
namespace v9 {
template <int RL, int SY>
struct KLowSI : KLowS<RL, SY> {
  static constexpr bool IDBL = true;
};
template <int RL, int SY>
struct KHighSI2 : KHighS<RL, SY> {
  static constexpr bool IDBL = true;
};
}  // namespace v9
sg_status exp_SIDBL(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                    cudaStream_t s) {
  using namespace v9;
  return run<KLowSI<6, 9>, KLowSI<4, 9>, KHighSI2<4, 9>, 256, 2, 128, 3>(L, a, x, p, m, y, s);
}
}  // namespace sg
