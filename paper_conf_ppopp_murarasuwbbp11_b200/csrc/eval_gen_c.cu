// eval_gen_c.cu -- instantiations of the generic evaluation kernel (eval_gen.cuh) for D = 9, 10.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_gen.cuh"

namespace sg {

bool launch_gen_c(int d, int n, bool f64, const void* a, const void* x, const uint32_t* p, uint64_t m, void* y,
                  cudaStream_t s, sg_status* st, const GenPart& pt) {
  switch (d) {
    case 9:
      *st = f64 ? gen::launch_gen<double, 9>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 9>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 10:
      *st = f64 ? gen::launch_gen<double, 10>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 10>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    default:
      return false;
  }
}

}  // namespace sg
