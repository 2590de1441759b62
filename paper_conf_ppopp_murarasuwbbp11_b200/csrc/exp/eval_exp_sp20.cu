// SP20 / SP20B: support-enumeration evaluation (eval_sparse.cuh) at d = 20, n <= 6, two CTA shapes
#include "eval_sparse.cuh"

namespace sg {
sg_status exp_SP20(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                   cudaStream_t s) {
  return sparse::launch<double, 20, 6, 64, 4>(L, a, x, p, m, y, s);
}
sg_status exp_SP20B(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                    cudaStream_t s) {
  return sparse::launch<double, 20, 6, 32, 8>(L, a, x, p, m, y, s);
}
}  // namespace sg
