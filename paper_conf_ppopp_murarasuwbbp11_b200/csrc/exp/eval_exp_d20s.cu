// D20S19 / D20S18 / D20S17: cfg5 (d = 20, n <= 6, S0 knob) with a CTA barrier at every level step of
// dimension 19 / 18 / 17 (one launch, 128 x 3 as the product)
#include "../eval_trie.cuh"

namespace sg {
template <int SY>
struct KnobsS0Y : trie::KnobsS0 {
  static constexpr int SYNC = SY;
};
#define SG_D20S(name, SY)                                                                                   \
  sg_status name(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y, \
                 cudaStream_t s) {                                                                          \
    return trie::launch_range<double, 20, 6, 128, 3, 0, 5, KnobsS0Y<SY>>(L, a, x, p, m, y, s);             \
  }
SG_D20S(exp_D20S19, 19)
SG_D20S(exp_D20S18, 18)
SG_D20S(exp_D20S17, 17)
}  // namespace sg
