// boundary.cu -- SURVEY 8(f) NEXT-2: sparse grids with non-zero boundary (Sec. 4.4, P:L461-L463;
// Fig. 7).  "The boundary of a d-dimensional sparse grid is composed of lower-dimensional,
// zero-boundary sparse grids for which we already have an efficient data structure": a grid with boundary
// is a list of FACES (S, c) -- S the free dimensions, c the values (0 / 1) of the fixed ones -- each
// carrying the |S|-dimensional zero-boundary grid of level n in the paper's compact layout, grouped by
// dimensionality (interior first, corners last; reading G20, include/sg.h).
//
//   hierarchization: one pass per dimension t; every face with t free runs the pole-family kernel of
//   hier_kernels.cu on its own |S|-dimensional layout, with the 1D parents that fall on the boundary read
//   from the two faces that fix t to 0 and 1 (for the family's subspace l_{-t}, a contiguous block of
//   2^{|l_{-t}|} values there, one per pole); those faces have t fixed and do not change in pass t;
//   evaluation: f_s(x) = sum_faces prod_{t fixed} b_{c_t}(x_t) f_face(x_S), b_0 = 1 - x, b_1 = x on [0,1];
//   each face's f_face is the ordinary zero-boundary evaluation path (sg_evaluate on the |S|-dimensional
//   grid, Morton order and the trie kernels) at the projected queries, accumulated with its weight.
#include <stdlib.h>
#include <string.h>

#include <new>
#include <vector>

#include "common.cuh"

struct sg_bgrid_s {
  int d, n, device;
  uint64_t N;
  struct Face {
    uint32_t mask, bits;  // free dimensions; values of the fixed ones (bit k = the k-th fixed dimension)
    int j;                // |S|
    uint64_t first, count;
  };
  std::vector<Face> faces;
  sg_grid sub[SG_MAX_D + 1] = {};  // the j-dimensional zero-boundary grids, j = 1..d
  // hierarchization tables per (j, local dimension): families with |l_{-t}| <= n-1 (the single-block ones
  // change too: their level-0 points have boundary parents)
  struct Tab {
    uint64_t F = 0;
    uint32_t* info = nullptr;    // [F]: s | suf << 8
    uint32_t* first = nullptr;   // [F]: first block base of the family
    uint64_t* bases = nullptr;   // block bases (face-local)
    uint64_t* bbase = nullptr;   // [F]: base of subspace l_{-t} in the (j-1)-dimensional face (local)
  };
  std::vector<Tab> tabs;  // index j * SG_MAX_D + t
  bool dev_ok = false;    // tables built (a CUDA device was present at sg_bcreate)
};

namespace sg {

namespace {

constexpr int kThreads = 256;

template <typename T>
__global__ void __launch_bounds__(kThreads) k_hier_family_b(int n, const uint32_t* __restrict__ info,
                                                            const uint32_t* __restrict__ first,
                                                            const uint64_t* __restrict__ bases,
                                                            const uint64_t* __restrict__ bbase, T* __restrict__ v,
                                                            const T* __restrict__ v0, const T* __restrict__ v1) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* fam = reinterpret_cast<T*>(smem_raw);
  __shared__ uint64_t base[SG_MAX_N];
  const uint32_t w0 = __ldg(info + blockIdx.x), f0 = __ldg(first + blockIdx.x);
  const int s = (int)(w0 & 0xff), suf = (int)(w0 >> 8), L = n - s;
  if ((int)threadIdx.x < L) base[threadIdx.x] = __ldg(bases + f0 + threadIdx.x);
  __syncthreads();
  const uint32_t two_s = 1u << s;
  const uint32_t E = ((1u << L) - 1u) << s;  // the family: block k at shared offset 2^{s+k} - 2^s
  T* b0 = fam + E;                            // boundary values of the poles at x_t = 0 and x_t = 1
  T* b1 = b0 + two_s;
  const uint64_t bb = __ldg(bbase + blockIdx.x);
  for (uint32_t w = threadIdx.x; w < E + 2 * two_s; w += blockDim.x) {
    T val;
    if (w < E) {
      const uint32_t p = w + two_s;
      const int k = 31 - __clz(p) - s;
      val = v[base[k] + (p - (1u << (s + k)))];
    } else if (w < E + two_s) {
      val = v0[bb + (w - E)];
    } else {
      val = v1[bb + (w - E - two_s)];
    }
    fam[w] = val;
  }
  __syncthreads();
  const uint32_t lomask = (1u << suf) - 1u;
  for (uint32_t w = threadIdx.x; w < E; w += blockDim.x) {
    const uint32_t p = w + two_s;
    const int k = 31 - __clz(p) - s;
    const uint32_t wl = p - (1u << (s + k));
    const uint32_t lo = wl & lomask;
    const uint32_t c = (wl >> suf) & ((1u << k) - 1u);
    const uint32_t hi = wl >> (suf + k);
    const uint32_t pole = (hi << suf) | lo;  // the pole's position in block 0 / in the boundary blocks
    T vl, vr;
    if (c != 0) {
      const int b = __ffs(c) - 1;
      const int kp = k - 1 - b;
      const uint32_t cp = (c >> b) >> 1;
      vl = fam[(((1u << kp) - 1u) << s) + ((((hi << kp) + cp) << suf) | lo)];
    } else {
      vl = b0[pole];  // the left parent is the boundary point x_t = 0
    }
    if (c + 1 != (1u << k)) {
      const int b = __ffs(c + 1) - 1;
      const int kp = k - 1 - b;
      const uint32_t cp = ((c + 1) >> b) >> 1;
      vr = fam[(((1u << kp) - 1u) << s) + ((((hi << kp) + cp) << suf) | lo)];
    } else {
      vr = b1[pole];  // the right parent is the boundary point x_t = 1
    }
    v[base[k] + wl] = fam[w] - (vl + vr) / T(2);
  }
}

// coordinates of a face's points embedded in d dimensions
template <typename T>
__global__ void __launch_bounds__(kThreads) k_embed(const T* __restrict__ xf, uint64_t count, int d, uint32_t mask,
                                                    uint32_t bits, T* __restrict__ x) {
  for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < count; p += (uint64_t)gridDim.x * blockDim.x) {
    int k = 0, kf = 0;
    for (int t = 0; t < d; ++t) {
      if (mask >> t & 1u) x[p * d + t] = xf[p * __popc(mask) + k++];
      else x[p * d + t] = (T)((bits >> kf++) & 1u);
    }
  }
}

// queries projected onto a face's free dimensions
template <typename T>
__global__ void __launch_bounds__(kThreads) k_project(const T* __restrict__ x, uint64_t m, int d, uint32_t mask,
                                                      T* __restrict__ xs) {
  const int j = __popc(mask);
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < m; q += (uint64_t)gridDim.x * blockDim.x) {
    int k = 0;
    for (int t = 0; t < d; ++t)
      if (mask >> t & 1u) xs[q * j + k++] = x[q * d + t];
  }
}

// y += prod_{t fixed} b_{c_t}(x_t) * (yf or the corner's surplus); weight 0 outside [0,1]^d, NaN propagates
template <typename T>
__global__ void __launch_bounds__(kThreads) k_face_axpy(const T* __restrict__ x, uint64_t m, int d, uint32_t mask,
                                                        uint32_t bits, const T* __restrict__ yf,
                                                        const T* __restrict__ corner, T* __restrict__ y) {
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < m; q += (uint64_t)gridDim.x * blockDim.x) {
    double w = 1.0;
    bool inside = true, bad = false;
    int kf = 0;
    for (int t = 0; t < d; ++t) {
      const double xt = (double)x[q * d + t];
      bad |= isnan(xt);
      inside &= (xt >= 0.0 && xt <= 1.0);
      if (!(mask >> t & 1u)) w *= ((bits >> kf++) & 1u) ? xt : 1.0 - xt;
    }
    const double f = corner ? (double)corner[0] : (double)yf[q];
    if (bad) y[q] = (T)NAN;
    else if (inside) y[q] = (T)((double)y[q] + w * f);
  }
}

unsigned grid_for(uint64_t n) {
  uint64_t b = (n + kThreads - 1) / kThreads;
  if (b > (uint64_t)kNumSMs * 32) b = (uint64_t)kNumSMs * 32;
  return (unsigned)(b ? b : 1);
}

}  // namespace

}  // namespace sg

using namespace sg;

static inline size_t dt_size(sg_dtype dt) { return dt == SG_F64 ? 8 : 4; }

static uint32_t fixed_bit_insert(uint32_t mask, uint32_t bits, int t, int val) {
  // bits of the face that fixes t (to val) in addition to the fixed dimensions of `mask`
  uint32_t out = 0;
  int kin = 0, kout = 0;
  for (int u = 0; u < 32; ++u) {
    const bool was_fixed = !(mask >> u & 1u);
    if (u == t) {
      out |= (uint32_t)val << kout++;
    } else if (was_fixed) {
      out |= ((bits >> kin++) & 1u) << kout++;
    }
  }
  return out;
}

static int face_index(const sg_bgrid_s* g, uint32_t mask, uint32_t bits) {
  for (size_t f = 0; f < g->faces.size(); ++f)
    if (g->faces[f].mask == mask && g->faces[f].bits == bits) return (int)f;
  return -1;
}

// host-built family tables for the j-dimensional face layout, local dimension t
static sg_status build_tab(sg_bgrid_s* g, int j, int t, sg_bgrid_s::Tab* tab) {
  const int n = g->n;
  // host layouts of the j- and (j-1)-dimensional face grids
  const sg::Layout* LJ = &g->sub[j]->L;
  const sg::Layout* LJ1 = j >= 2 ? &g->sub[j - 1]->L : nullptr;
  std::vector<uint32_t> info, first;
  std::vector<uint64_t> bases, bbase;
  // enumerate the (j-1)-dimensional level vectors with sum <= n-1 (the family keys)
  std::vector<int32_t> w(j > 1 ? j - 1 : 1, 0);
  const int dm = j - 1;
  std::vector<int32_t> lv(j);
  auto visit = [&](const std::vector<int32_t>& wv) {
    int s = 0, suf = 0;
    for (int u = 0, k = 0; u < j; ++u) {
      lv[u] = (u == t) ? 0 : wv[k++];
      s += lv[u];
      if (u > t) suf += lv[u];
    }
    info.push_back((uint32_t)s | ((uint32_t)suf << 8));
    first.push_back((uint32_t)bases.size());
    for (int k = 0; k < n - s; ++k) {
      lv[t] = k;
      bases.push_back(LJ->off[s + k] + (subspace_rank(*LJ, lv.data()) << (s + k)));
    }
    lv[t] = 0;
    if (dm == 0) {
      bbase.push_back(0);  // the corner: a single value
    } else {
      std::vector<int32_t> lm;
      for (int u = 0; u < j; ++u)
        if (u != t) lm.push_back(lv[u]);
      bbase.push_back(LJ1->off[s] + (subspace_rank(*LJ1, lm.data()) << s));
    }
  };
  if (dm == 0) {
    visit(w);
  } else {
    // odometer over dm components with sum <= n-1
    std::vector<int32_t> c(dm, 0);
    while (true) {
      visit(c);
      int k = 0;
      while (k < dm) {
        c[k]++;
        int sum = 0;
        for (int u = 0; u < dm; ++u) sum += c[u];
        if (sum <= n - 1) break;
        c[k] = 0;
        ++k;
      }
      if (k == dm) break;
    }
  }
  tab->F = info.size();
  cudaError_t e = cudaMalloc(&tab->info, info.size() * 4);
  if (e == cudaSuccess) e = cudaMalloc(&tab->first, first.size() * 4);
  if (e == cudaSuccess) e = cudaMalloc(&tab->bases, bases.size() * 8);
  if (e == cudaSuccess) e = cudaMalloc(&tab->bbase, bbase.size() * 8);
  if (e == cudaSuccess) e = cudaMemcpy(tab->info, info.data(), info.size() * 4, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(tab->first, first.data(), first.size() * 4, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(tab->bases, bases.data(), bases.size() * 8, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(tab->bbase, bbase.data(), bbase.size() * 8, cudaMemcpyHostToDevice);
  return e == cudaSuccess ? SG_OK : cuda_fail(e, "sg_bcreate: hierarchization tables");
}

extern "C" {

sg_status sg_bcreate(int32_t d, int32_t n, sg_bgrid* out, uint64_t* num_points) {
  if (!out) return SG_ERR_ARG;
  *out = nullptr;
  if (d < 1 || d > 12 || n < 1 || n > 14) {
    set_error("sg_bcreate: need 1 <= d <= 12 and 1 <= n <= 14 (got d=%d, n=%d)", d, n);
    return SG_ERR_ARG;
  }
  sg_bgrid_s* g = new (std::nothrow) sg_bgrid_s();
  if (!g) return SG_ERR_NOMEM;
  g->d = d;
  g->n = n;
  g->device = -1;
  cudaGetDevice(&g->device);
  sg_status st = SG_OK;
  for (int j = 1; j <= d && st == SG_OK; ++j) st = sg_create(j, n, &g->sub[j], nullptr);
  if (st != SG_OK) {
    sg_bdestroy(g);
    return st;
  }
  // faces in layout order: dimensionality j = d..0, free mask ascending, fixed values ascending
  uint64_t pos = 0;
  for (int j = d; j >= 0; --j)
    for (uint32_t mask = 0; mask < (1u << d); ++mask) {
      if (__builtin_popcount(mask) != j) continue;
      for (uint32_t bits = 0; bits < (1u << (d - j)); ++bits) {
        uint64_t cnt = 1;
        if (j > 0) {
          sg_layout lay;
          sg_get_layout(g->sub[j], &lay);
          cnt = lay.num_points;
        }
        g->faces.push_back({mask, bits, j, pos, cnt});
        pos += cnt;
      }
    }
  g->N = pos;
  g->tabs.resize((size_t)(d + 1) * SG_MAX_D);
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) == cudaSuccess && ndev > 0 && n >= 1) {
    for (int j = 1; j <= d && st == SG_OK; ++j)
      for (int t = 0; t < j && st == SG_OK; ++t) st = build_tab(g, j, t, &g->tabs[(size_t)j * SG_MAX_D + t]);
    g->dev_ok = st == SG_OK;
  } else {
    cudaGetLastError();
  }
  if (st != SG_OK) {
    sg_bdestroy(g);
    return st;
  }
  *out = g;
  if (num_points) *num_points = g->N;
  return SG_OK;
}

sg_status sg_bdestroy(sg_bgrid g) {
  if (!g) return SG_OK;
  for (auto& t : g->tabs) {
    cudaFree(t.info);
    cudaFree(t.first);
    cudaFree(t.bases);
    cudaFree(t.bbase);
  }
  for (int j = 1; j <= g->d; ++j)
    if (g->sub[j]) sg_destroy(g->sub[j]);
  delete g;
  return SG_OK;
}

sg_status sg_bface(sg_bgrid g, uint32_t face, uint32_t* free_mask, uint32_t* fixed_bits, uint64_t* first,
                   uint64_t* count) {
  if (!g || !free_mask || !fixed_bits || !first || !count) return SG_ERR_ARG;
  if (face >= g->faces.size()) {
    set_error("sg_bface: face %u >= 3^d = %zu", face, g->faces.size());
    return SG_ERR_RANGE;
  }
  const auto& f = g->faces[face];
  *free_mask = f.mask;
  *fixed_bits = f.bits;
  *first = f.first;
  *count = f.count;
  return SG_OK;
}

sg_status sg_bcoords_device(sg_bgrid g, void* d_x, sg_dtype dt, void* stream) {
  if (!g || !d_x) return SG_ERR_ARG;
  if (!g->dev_ok) {
    set_error("boundary grid has no device (created without a GPU)");
    return SG_ERR_NODEV;
  }
  if (dt != SG_F64 && dt != SG_F32) return SG_ERR_DTYPE;
  NvtxRange nvtx("sg_bcoords_device");
  cudaStream_t s = (cudaStream_t)stream;
  const size_t es = dt_size(dt);
  const int d = g->d;
  void* tmp = nullptr;
  uint64_t maxc = 1;
  for (const auto& f : g->faces) maxc = f.count > maxc ? f.count : maxc;
  cudaError_t e = cudaMallocAsync(&tmp, maxc * d * es, s);
  if (e != cudaSuccess) return cuda_fail(e, "sg_bcoords_device: cudaMallocAsync");
  sg_status st = SG_OK;
  for (const auto& f : g->faces) {
    if (f.j > 0) st = sg_grid_coords_device(g->sub[f.j], 0, f.count, tmp, dt, stream);
    if (st != SG_OK) break;
    if (dt == SG_F64)
      k_embed<double><<<grid_for(f.count), kThreads, 0, s>>>((const double*)tmp, f.count, d, f.mask, f.bits,
                                                             (double*)d_x + f.first * d);
    else
      k_embed<float><<<grid_for(f.count), kThreads, 0, s>>>((const float*)tmp, f.count, d, f.mask, f.bits,
                                                            (float*)d_x + f.first * d);
    st = launched("k_embed", dt == SG_F64 ? (const void*)k_embed<double> : (const void*)k_embed<float>);
    if (st != SG_OK) break;
  }
  cudaFreeAsync(tmp, s);
  return st;
}

sg_status sg_bhierarchize(sg_bgrid g, void* d_values, sg_dtype dt, void* stream) {
  if (!g || !d_values) return SG_ERR_ARG;
  if (!g->dev_ok) {
    set_error("boundary grid has no device (created without a GPU)");
    return SG_ERR_NODEV;
  }
  if (dt != SG_F64 && dt != SG_F32) return SG_ERR_DTYPE;
  NvtxRange nvtx("sg_bhierarchize");
  cudaStream_t s = (cudaStream_t)stream;
  const size_t es = dt_size(dt);
  const int n = g->n;
  int dev = 0, max_smem = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const size_t fam_bytes = ((((size_t)1 << n) - 1) + 2 * ((size_t)1 << (n - 1))) * es;
  if (fam_bytes + 512 > (size_t)max_smem) {
    set_error("sg_bhierarchize: level n=%d needs %zu B of shared memory per pole family", n, fam_bytes);
    return SG_ERR_ARG;
  }
  static std::atomic<uint64_t> done64{0}, done32{0};
  sg_status st = dt == SG_F64 ? set_smem_attr(k_hier_family_b<double>, done64, (size_t)max_smem - 512, -1, "attr")
                              : set_smem_attr(k_hier_family_b<float>, done32, (size_t)max_smem - 512, -1, "attr");
  if (st != SG_OK) return st;
  char* v = (char*)d_values;
  for (int t = 0; t < g->d; ++t) {
    for (const auto& f : g->faces) {
      if (!(f.mask >> t & 1u)) continue;  // t fixed on this face: its points are unchanged in pass t
      // t's position among the face's free dimensions, and the two faces that fix t to 0 / 1
      const int tl = __builtin_popcount(f.mask & ((1u << t) - 1u));
      const uint32_t m2 = f.mask & ~(1u << t);
      const int f0 = face_index(g, m2, fixed_bit_insert(f.mask, f.bits, t, 0));
      const int f1 = face_index(g, m2, fixed_bit_insert(f.mask, f.bits, t, 1));
      if (f0 < 0 || f1 < 0) return SG_ERR_ARG;
      const auto& tab = g->tabs[(size_t)f.j * SG_MAX_D + tl];
      const size_t smem = ((((size_t)1 << n) - 1) + 2 * ((size_t)1 << (n - 1))) * es;
      if (dt == SG_F64)
        k_hier_family_b<double><<<(unsigned)tab.F, kThreads, smem, s>>>(
            n, tab.info, tab.first, tab.bases, tab.bbase, (double*)(v + f.first * es),
            (const double*)(v + g->faces[f0].first * es), (const double*)(v + g->faces[f1].first * es));
      else
        k_hier_family_b<float><<<(unsigned)tab.F, kThreads, smem, s>>>(
            n, tab.info, tab.first, tab.bases, tab.bbase, (float*)(v + f.first * es),
            (const float*)(v + g->faces[f0].first * es), (const float*)(v + g->faces[f1].first * es));
      st = launched("k_hier_family_b", dt == SG_F64 ? (const void*)k_hier_family_b<double> : (const void*)k_hier_family_b<float>);
      if (st != SG_OK) return st;
    }
  }
  return SG_OK;
}

sg_status sg_bevaluate(sg_bgrid g, const void* d_alpha, const void* d_x, uint64_t m, void* d_y, sg_dtype dt,
                       void* stream) {
  if (!g || !d_alpha || !d_x || !d_y) return SG_ERR_ARG;
  if (!g->dev_ok) {
    set_error("boundary grid has no device (created without a GPU)");
    return SG_ERR_NODEV;
  }
  if (dt != SG_F64 && dt != SG_F32) return SG_ERR_DTYPE;
  if (m == 0) return SG_OK;
  NvtxRange nvtx("sg_bevaluate");
  cudaStream_t s = (cudaStream_t)stream;
  const size_t es = dt_size(dt);
  const int d = g->d;
  void *xs = nullptr, *yf = nullptr;
  cudaError_t e = cudaMallocAsync(&xs, m * (d > 1 ? d - 1 : 1) * es, s);
  if (e == cudaSuccess) e = cudaMallocAsync(&yf, m * es, s);
  if (e != cudaSuccess) return cuda_fail(e, "sg_bevaluate: cudaMallocAsync");
  sg_status st = SG_OK;
  const char* a = (const char*)d_alpha;
  for (const auto& f : g->faces) {
    if (f.j == d) {  // the interior: the zero-boundary path writes y
      st = sg_evaluate(g->sub[d], a + f.first * es, d_x, m, d_y, dt, 0, nullptr, 0, stream);
      if (st != SG_OK) break;
      continue;
    }
    const void* corner = nullptr;
    if (f.j > 0) {
      if (dt == SG_F64) k_project<double><<<grid_for(m), kThreads, 0, s>>>((const double*)d_x, m, d, f.mask, (double*)xs);
      else k_project<float><<<grid_for(m), kThreads, 0, s>>>((const float*)d_x, m, d, f.mask, (float*)xs);
      st = launched("k_project", dt == SG_F64 ? (const void*)k_project<double> : (const void*)k_project<float>);
      if (st == SG_OK) st = sg_evaluate(g->sub[f.j], a + f.first * es, xs, m, yf, dt, 0, nullptr, 0, stream);
      if (st != SG_OK) break;
    } else {
      corner = a + f.first * es;
    }
    if (dt == SG_F64)
      k_face_axpy<double><<<grid_for(m), kThreads, 0, s>>>((const double*)d_x, m, d, f.mask, f.bits, (const double*)yf,
                                                           (const double*)corner, (double*)d_y);
    else
      k_face_axpy<float><<<grid_for(m), kThreads, 0, s>>>((const float*)d_x, m, d, f.mask, f.bits, (const float*)yf,
                                                          (const float*)corner, (float*)d_y);
    st = launched("k_face_axpy", dt == SG_F64 ? (const void*)k_face_axpy<double> : (const void*)k_face_axpy<float>);
    if (st != SG_OK) break;
  }
  cudaFreeAsync(xs, s);
  cudaFreeAsync(yf, s);
  return st;
}

}  // extern "C"
