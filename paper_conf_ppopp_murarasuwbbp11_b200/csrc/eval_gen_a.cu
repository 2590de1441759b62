// eval_gen_a.cu -- instantiations of the generic evaluation kernel (eval_gen.cuh) for D = 1, 2, 3, 4, 5.
// Split across files only so that nvcc compiles them in parallel.
#include "eval_gen.cuh"

namespace sg {

bool launch_gen_a(int d, int n, bool f64, const void* a, const void* x, const uint32_t* p, uint64_t m, void* y,
                  cudaStream_t s, sg_status* st, const GenPart& pt) {
  switch (d) {
    case 1:
      *st = f64 ? gen::launch_gen<double, 1>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 1>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 2:
      *st = f64 ? gen::launch_gen<double, 2>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 2>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 3:
      *st = f64 ? gen::launch_gen<double, 3>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 3>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 4:
      *st = f64 ? gen::launch_gen<double, 4>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 4>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    case 5:
      *st = f64 ? gen::launch_gen<double, 5>((const double*)a, (const double*)x, p, m, n, (double*)y, s, pt.j0, pt.v0,
                                               pt.j1, pt.v1, pt.b0, pt.accumulate)
                : gen::launch_gen<float, 5>((const float*)a, (const float*)x, p, m, n, (float*)y, s, pt.j0, pt.v0,
                                              pt.j1, pt.v1, pt.b0, pt.accumulate);
      return true;
    default:
      return false;
  }
}

}  // namespace sg
