// plane_kernels.cu -- SURVEY 8(f) NEXT-3: the visualization slice path.  The paper's motivating
// application is interactive visualization of compressed simulation data (Fig. 1):
// decompression "at arbitrary locations" -- here every pixel of a 2D slice through the domain.
//
// sg_evaluate_plane renders a width x height image of f_s on the plane
//     x(a, b) = origin + (a + 1/2) du + (b + 1/2) dv      (pixel column a, row b; image row-major)
// without a host query array: k_plane_coords writes the pixel coordinates (row-major) and the order in
// which the evaluation kernel visits the pixels, then the ordinary evaluation kernels run with that order
// (the `perm` of sg_evaluate): each warp takes an 8 x 4 pixel tile and the tiles follow a 2D Morton
// curve (order 1), or the image's row-major order (order 0).  A slice has no spatial sort to do -- its
// pixels are already on a 2D lattice -- so the tile order replaces row a1 ("compare row-major
// image order with 2D-Morton 8x4 warp tiles").
#include "common.cuh"

namespace sg {

namespace {

constexpr int kThreads = 256;

struct PlaneArgs {
  double o[SG_MAX_D], u[SG_MAX_D], v[SG_MAX_D];
};

// 2D Morton index -> (tx, ty): even bits to x, odd bits to y
__device__ __forceinline__ uint32_t compact1by1(uint32_t z) {
  z &= 0x55555555u;
  z = (z ^ (z >> 1)) & 0x33333333u;
  z = (z ^ (z >> 2)) & 0x0f0f0f0fu;
  z = (z ^ (z >> 4)) & 0x00ff00ffu;
  z = (z ^ (z >> 8)) & 0x0000ffffu;
  return z;
}

template <typename T>
__global__ void __launch_bounds__(kThreads) k_plane_coords(PlaneArgs pa, int d, uint32_t w, uint32_t h, int order,
                                                           uint32_t tiles_x, int kx, int ky,
                                                           T* __restrict__ x, uint32_t* __restrict__ perm) {
  const uint64_t m = (uint64_t)w * h;
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < m; q += (uint64_t)gridDim.x * blockDim.x) {
    // pixel of the row-major position q: its coordinates, written in image order
    const uint32_t a = (uint32_t)(q % w), b = (uint32_t)(q / w);
    for (int t = 0; t < d; ++t) {
      // x_t = fl(fl(o_t + (a+1/2) u_t) + (b+1/2) v_t): fixed rounding (no contraction)
      const double v = __dadd_rn(__dadd_rn(pa.o[t], __dmul_rn((double)a + 0.5, pa.u[t])), __dmul_rn((double)b + 0.5, pa.v[t]));
      x[q * d + t] = (T)v;
    }
    // the q-th pixel the evaluation visits
    uint32_t pa_, pb_;
    if (order == 0) {
      pa_ = a;
      pb_ = b;
    } else {
      // warp tile of 8 x 4 pixels; tiles along a 2D Morton curve when the tile grid is 2^kx x 2^ky
      // (the low 2 min(kx, ky) bits interleaved, the rest to the longer side), else row-major tiles
      const uint32_t lane = (uint32_t)(q & 31u), tile = (uint32_t)(q >> 5);
      uint32_t tx, ty;
      if (kx >= 0 && ky >= 0) {
        const int k = kx < ky ? kx : ky;
        const uint32_t lowz = tile & ((1u << (2 * k)) - 1u), hi = tile >> (2 * k);
        tx = compact1by1(lowz);
        ty = compact1by1(lowz >> 1);
        if (kx > ky) tx |= hi << k;
        else ty |= hi << k;
      } else {
        tx = tile % tiles_x;
        ty = tile / tiles_x;
      }
      pa_ = tx * 8 + (lane & 7u);
      pb_ = ty * 4 + (lane >> 3);
    }
    perm[q] = pb_ * w + pa_;
  }
}

}  // namespace

size_t plane_workspace_bytes(int d, uint64_t m, size_t elem) {
  return ((m * (uint64_t)d * elem + 255) & ~(uint64_t)255) + ((m * 4 + 255) & ~(uint64_t)255);
}

sg_status launch_plane(const sg_grid_s* g, const void* alpha, const double* origin, const double* du, const double* dv,
                       uint32_t width, uint32_t height, void* img, sg_dtype dt, uint32_t order, void* ws,
                       cudaStream_t s) {
  const int d = g->L.d;
  const uint64_t m = (uint64_t)width * height;
  PlaneArgs pa;
  for (int t = 0; t < d; ++t) {
    pa.o[t] = origin[t];
    pa.u[t] = du[t];
    pa.v[t] = dv[t];
  }
  const size_t elem = dt == SG_F64 ? 8 : 4;
  char* p = (char*)ws;
  void* x = p;
  uint32_t* perm = (uint32_t*)(p + ((m * (uint64_t)d * elem + 255) & ~(uint64_t)255));
  // tile order needs whole 8 x 4 tiles
  const int ord = (order == 1 && width % 8 == 0 && height % 4 == 0) ? 1 : 0;
  const uint32_t tiles_x = width / 8, tiles_y = height / 4;
  auto log2_exact = [](uint32_t v) { return (v && !(v & (v - 1))) ? 31 - __builtin_clz(v) : -1; };
  const int kx = log2_exact(tiles_x), ky = log2_exact(tiles_y);
  uint64_t blocks = (m + kThreads - 1) / kThreads;
  if (blocks > (uint64_t)kNumSMs * 32) blocks = (uint64_t)kNumSMs * 32;
  if (dt == SG_F64)
    k_plane_coords<double><<<(unsigned)blocks, kThreads, 0, s>>>(pa, d, width, height, ord, tiles_x, kx, ky,
                                                                  (double*)x, perm);
  else
    k_plane_coords<float><<<(unsigned)blocks, kThreads, 0, s>>>(pa, d, width, height, ord, tiles_x, kx, ky,
                                                                 (float*)x, perm);
  sg_status st = launched("k_plane_coords", dt == SG_F64 ? (const void*)k_plane_coords<double> : (const void*)k_plane_coords<float>);
  if (st != SG_OK) return st;
  return launch_evaluate(g, alpha, x, perm, m, img, dt, 0, s);
}

}  // namespace sg
