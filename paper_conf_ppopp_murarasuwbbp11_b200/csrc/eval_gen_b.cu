// eval_gen_b.cu -- instantiations of the generic evaluation kernel (eval_gen.cuh) for D = 6, 7, 8.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_gen.cuh"

namespace sg {

bool launch_gen_b(int d, int n, bool f64, const void* a, const void* x, const uint32_t* p, uint64_t m, void* y,
                  cudaStream_t s, sg_status* st, const GenPart& pt) {
  switch (d) {
    case 6:
      *st = f64 ? gen::launch_gen<double, 6>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 6>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 7:
      *st = f64 ? gen::launch_gen<double, 7>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 7>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 8:
      *st = f64 ? gen::launch_gen<double, 8>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 8>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    default:
      return false;
  }
}

}  // namespace sg
