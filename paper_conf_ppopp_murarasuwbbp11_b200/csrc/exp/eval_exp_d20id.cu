// D20ID: cfg5 (d = 20, n <= 6, S0 knob) with the dimension-4 hats by doubling (IDBL: 5 fewer shared-memory
// rows per 128 queries; the d = 20 launch holds 69 rows, 207 KB per SM, leaving ~28 KB of L1)
#include "../eval_trie.cuh"

namespace sg {
struct KnobsS0ID : trie::KnobsS0 {
  static constexpr bool IDBL = true;
};
sg_status exp_D20ID(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                    cudaStream_t s) {
  return trie::launch_range<double, 20, 6, 128, 3, 0, 5, KnobsS0ID>(L, a, x, p, m, y, s);
}
}  // namespace sg
