// LIDBL: the v9.2 product with the dimension-4 hats of the large-block launches by doubling (IDBL: 10 fewer
// shared-memory rows per 128 queries, so more L1 for the launches that run at 60% L1 hits)
#include "exp_sync.cuh"
namespace sg {
namespace v9 {
template <int RL, int SY>
struct KHighSI : KHighS<RL, SY> {
  static constexpr bool IDBL = true;
};
}  // namespace v9
sg_status exp_LIDBL(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                    cudaStream_t s) {
  using namespace v9;
  return run<KLowS<6, 9>, KLowS<4, 9>, KHighSI<4, 9>, 256, 2, 128, 3>(L, a, x, p, m, y, s);
}
}  // namespace sg
