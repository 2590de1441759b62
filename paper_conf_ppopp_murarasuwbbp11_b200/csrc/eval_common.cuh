// eval_common.cuh -- per-dimension 1D quantities of the evaluation (row a2).
#pragma once
#include <math.h>
#include <stdint.h>

namespace sg {

// Hat value phi_{l,i}(x) of the cell of x at level l (0-based), and that cell
// k (i = 2k+1).  P:L87: phi_{l,i}(x) = max(0, 1 - |2^{l+1} x - i|).  With
// y = 2^l x, k = clamp(floor(y), 0, 2^l - 1) (reading G8) and u = y - k this is
// max(0, 2 min(u, 1 - u)), exact in floating point: y is a power-of-two
// scaling, u is exact (Sterbenz for k >= 1), and 1 - u is exact whenever it is
// the smaller of the two.  Outside [0,1] the clamped cell gives u < 0 or
// u > 1 and therefore 0; NaN is handled by the caller.
template <typename T>
__device__ __forceinline__ T hat_cell(T x, int l, uint32_t& cell) {
  const T y = x * (T)(1u << l);  // l <= 30
  T k = floor(y);
  const T top = (T)((1u << l) - 1u);
  k = k < T(0) ? T(0) : k;
  k = k > top ? top : k;
  cell = (uint32_t)k;
  const T u = y - k;
  const T w = T(1) - u;
  const T mn = u < w ? u : w;
  const T h = mn + mn;
  return h > T(0) ? h : T(0);
}

}  // namespace sg
