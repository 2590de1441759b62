// eval_gen_d.cu -- instantiations of the generic evaluation kernel (eval_gen.cuh) for D = 11, 12.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_gen.cuh"

namespace sg {

bool launch_gen_d(int d, int n, bool f64, const void* a, const void* x, const uint32_t* p, uint64_t m, void* y,
                  cudaStream_t s, sg_status* st, const GenPart& pt) {
  switch (d) {
    case 11:
      *st = f64 ? gen::launch_gen<double, 11>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 11>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 12:
      *st = f64 ? gen::launch_gen<double, 12>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 12>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    default:
      return false;
  }
}

}  // namespace sg
