// exp_sync.cuh -- EXPERIMENT (libsg_exp.so only): the v9 product with a CTA barrier at every level step of one
// outer dimension (Knobs::SYNC), in both launches of every group.
#pragma once
#include "exp_v9.cuh"

namespace sg {
namespace v9 {
template <int RL, int SY>
struct KLowS : KLow9<RL, false, true> {
  static constexpr int SYNC = SY;
};
template <int RL, int SY>
struct KHighS : KHighN<RL> {
  static constexpr int SYNC = SY;
};
}  // namespace v9
}  // namespace sg
#define SG_SYNC(name, SY)                                                                                      \
  namespace sg {                                                                                               \
  sg_status name(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,    \
                 cudaStream_t s) {                                                                             \
    using namespace v9;                                                                                        \
    return run<KLowS<6, SY>, KLowS<4, SY>, KHighS<4, SY>, 256, 2, 128, 3>(L, a, x, p, m, y, s);               \
  }                                                                                                            \
  }
// barrier only in the small-block (SYL) or only in the large-block (SYH) launches
#define SG_SYNC2(name, SYL, SYH)                                                                               \
  namespace sg {                                                                                               \
  sg_status name(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,    \
                 cudaStream_t s) {                                                                             \
    using namespace v9;                                                                                        \
    return run<KLowS<6, SYL>, KLowS<4, SYL>, KHighS<4, SYH>, 256, 2, 128, 3>(L, a, x, p, m, y, s);            \
  }                                                                                                            \
  }
