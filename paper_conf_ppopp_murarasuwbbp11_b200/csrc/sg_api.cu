// sg_api.cu -- the C ABI of libsg (include/sg.h): argument checking, handle
// management, host index maps, and dispatch to the CUDA launchers.
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>
#include <set>
#include <string>
#include <new>
#include <vector>

#include "common.cuh"

namespace sg {

std::atomic<uint64_t> g_launches{0};

static thread_local char t_err[512] = "";

// kernels launched since load (test instrumentation: sg_launched_kernels)
static std::mutex g_kern_mu;
static std::set<const void*> g_kernels;
void record_kernel(const void* func) {
  std::lock_guard<std::mutex> lk(g_kern_mu);
  g_kernels.insert(func);
}

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(t_err, sizeof(t_err), fmt, ap);
  va_end(ap);
}

// ---- profiling: event pairs recorded on the launching stream
static std::atomic<int> g_prof_on{0};
static std::mutex g_prof_mu;
struct ProfRec {
  cudaEvent_t a, b;
  int kind;
};
static std::vector<ProfRec> g_prof_pending;
static double g_prof_ms[2] = {0, 0};
static uint64_t g_prof_n[2] = {0, 0};

ProfScope::ProfScope(int kind_, cudaStream_t s_) : s(s_), kind(kind_) {
  if (!g_prof_on.load()) return;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a, s);
}

// fold finished event pairs into the totals (caller holds g_prof_mu)
static cudaError_t prof_fold(size_t keep) {
  cudaError_t st = cudaSuccess;
  const size_t n = g_prof_pending.size() > keep ? g_prof_pending.size() - keep : 0;
  for (size_t k = 0; k < n; ++k) {
    ProfRec& r = g_prof_pending[k];
    cudaError_t e = cudaEventSynchronize(r.b);
    float ms = 0.f;
    if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, r.a, r.b);
    if (e != cudaSuccess) st = e;
    g_prof_ms[r.kind] += ms;
    g_prof_n[r.kind] += 1;
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  g_prof_pending.erase(g_prof_pending.begin(), g_prof_pending.begin() + n);
  return st;
}

ProfScope::~ProfScope() {
  if (!a) return;
  cudaEventRecord(b, s);
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_prof_pending.push_back({a, b, kind});
  // bounded: beyond kProfMax outstanding pairs the oldest half is resolved (profiling mode only)
  constexpr size_t kProfMax = 4096;
  if (g_prof_pending.size() > kProfMax) prof_fold(kProfMax / 2);
}

sg_status cuda_fail(cudaError_t e, const char* what) {
  set_error("%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
  return SG_ERR_CUDA;
}

sg_status launch_eval_simple(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                             void* y, sg_dtype dt, cudaStream_t s);
#define SG_GEN_DECL(part)                                                                                      \
  bool launch_gen_##part(int d, int n, bool f64, const void* a, const void* x, const uint32_t* p, uint64_t m, \
                         void* y, cudaStream_t s, sg_status* st, const GenPart& pt);
SG_GEN_DECL(a) SG_GEN_DECL(b) SG_GEN_DECL(c) SG_GEN_DECL(d)
#undef SG_GEN_DECL

// the generic run-time-level kernel (eval_gen.cuh): d <= 12, n <= 12; 32-bit offsets
static sg_status launch_eval_gen(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm,
                                 uint64_t m, void* y, sg_dtype dt, cudaStream_t s, bool* handled,
                                 const GenPart& pt = GenPart()) {
  *handled = false;
  const int d = g->L.d, n = g->L.n;
  if (n > 12 || d > 12 || m > 0xffffffffull || g->L.N >= 0xffffffffull) return SG_OK;
  sg_status st = SG_OK;
  const bool f64 = dt == SG_F64;
  *handled = launch_gen_a(d, n, f64, alpha, x, perm, m, y, s, &st, pt) ||
             launch_gen_b(d, n, f64, alpha, x, perm, m, y, s, &st, pt) ||
             launch_gen_c(d, n, f64, alpha, x, perm, m, y, s, &st, pt) ||
             launch_gen_d(d, n, f64, alpha, x, perm, m, y, s, &st, pt);
  return st;
}

// ---- sharded grids: the layout cut into contiguous parts at (group j, level l_{d-1} = v)
// unit boundaries (whole groups for d <= 5, whose generic kernel has no separate top trie loop), each part
// holding about 1/parts of the subspaces (= of the evaluation work: one gather per subspace per query).
struct PartRange {
  GenPart gp;
  uint64_t first, count;
};
static void part_range(const Layout& L, uint32_t parts, uint32_t part, PartRange* out) {
  const int d = L.d, n = L.n;
  const bool fine = d >= 6;
  struct Unit {
    int j, v;
    uint64_t subs;
  };
  std::vector<Unit> units;  // in layout order: group j ascending, then l_{d-1} ascending (Alg. 3: slowest)
  for (int j = 0; j < n; ++j) {
    if (!fine) {
      units.push_back({j, -1, L.cnt[j]});
      continue;
    }
    for (int v = 0; v <= j; ++v) units.push_back({j, v, L.C(d - 2, j - v)});  // C(j-v+d-2, d-2) subspaces
  }
  // part p takes the units whose cumulative start lies in [p T / parts, (p+1) T / parts)
  const uint64_t lo = (uint64_t)((unsigned __int128)L.T * part / parts);
  const uint64_t hi = (uint64_t)((unsigned __int128)L.T * (part + 1) / parts);
  uint64_t cum = 0;
  int ua = -1, ub = -1;
  for (size_t u = 0; u < units.size(); ++u) {
    if (cum >= lo && cum < hi) {
      if (ua < 0) ua = (int)u;
      ub = (int)u;
    }
    cum += units[u].subs;
  }
  out->gp = GenPart();
  if (ua < 0) {  // empty part (more parts than units)
    out->gp.j0 = 1;
    out->gp.j1 = 0;
    out->first = out->count = 0;
    return;
  }
  auto unit_first = [&](int u) {  // index3(j) + (subspaces of group j before the unit) 2^j
    const int j = units[u].j;
    uint64_t before = 0;
    for (int w = u - 1; w >= 0 && units[w].j == j; --w) before += units[w].subs;
    return L.off[j] + (before << j);
  };
  const uint64_t first = unit_first(ua);
  const uint64_t last = unit_first(ub) + (units[ub].subs << units[ub].j);
  out->gp.j0 = units[ua].j;
  out->gp.v0 = fine ? units[ua].v : 0;
  out->gp.j1 = units[ub].j;
  out->gp.v1 = fine ? units[ub].v : 64;
  out->gp.b0 = (uint32_t)first;
  out->first = first;
  out->count = last - first;
}
sg_status launch_eval_trie(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                           void* y, sg_dtype dt, cudaStream_t s, bool* handled);

sg_status launch_evaluate(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                          void* y, sg_dtype dt, uint32_t flags, cudaStream_t s) {
  if (m == 0) return SG_OK;
  ProfScope prof(kProfEval, s);
  if (!(flags & SG_EVAL_GENERIC)) {
    bool handled = false;
    sg_status st = launch_eval_trie(g, alpha, x, perm, m, y, dt, s, &handled);
    if (handled || st != SG_OK) return st;
    st = launch_eval_gen(g, alpha, x, perm, m, y, dt, s, &handled);
    if (handled || st != SG_OK) return st;
  }
  return launch_eval_simple(g, alpha, x, perm, m, y, dt, s);
}

}  // namespace sg

using namespace sg;

static inline bool dtype_ok(sg_dtype dt) { return dt == SG_F64 || dt == SG_F32; }
static inline size_t dtype_size(sg_dtype dt) { return dt == SG_F64 ? 8 : 4; }

#define SG_CHECK_GRID(g)             \
  do {                               \
    if (!(g)) {                      \
      set_error("NULL grid handle"); \
      return SG_ERR_ARG;             \
    }                                \
  } while (0)

#define SG_CHECK_DEVICE(g)                                            \
  do {                                                                \
    if (!(g)->d_L) {                                                  \
      set_error("grid handle has no device (created without a GPU)"); \
      return SG_ERR_NODEV;                                            \
    }                                                                 \
  } while (0)

// Run device calls on the grid's device, restoring the caller's device after.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

extern "C" {

sg_status sg_create(int32_t d, int32_t n, sg_grid* out, uint64_t* num_points) {
  if (!out) {
    set_error("sg_create: out is NULL");
    return SG_ERR_ARG;
  }
  *out = nullptr;
  if (d < 1 || d > SG_MAX_D || n < 1 || n > SG_MAX_N) {
    set_error("sg_create: need 1 <= d <= %d and 1 <= n <= %d (got d=%d, n=%d)", SG_MAX_D, SG_MAX_N, d, n);
    return SG_ERR_ARG;
  }
  sg_grid_s* g = new (std::nothrow) sg_grid_s();
  if (!g) return SG_ERR_NOMEM;
  if (!build_layout(d, n, &g->L)) {
    delete g;
    set_error("sg_create: grid d=%d n=%d has >= 2^62 points", d, n);
    return SG_ERR_OVERFLOW;
  }
  g->device = -1;
  g->d_L = nullptr;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    // host-only handle: sg_get_layout / sg_gp2idx / sg_idx2gp work, device calls return SG_ERR_NODEV
    cudaGetLastError();
    set_error("sg_create: no CUDA device (%s); host-only handle", e == cudaSuccess ? "count 0" : cudaGetErrorString(e));
  } else {
    cudaGetDevice(&g->device);
    e = cudaMalloc((void**)&g->d_L, sizeof(Layout));
    if (e != cudaSuccess) {
      delete g;
      return cuda_fail(e, "sg_create: cudaMalloc");
    }
    e = cudaMemcpy(g->d_L, &g->L, sizeof(Layout), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      cudaFree(g->d_L);
      delete g;
      return cuda_fail(e, "sg_create: cudaMemcpy");
    }
  }
  *out = g;
  if (num_points) *num_points = g->L.N;
  return SG_OK;
}

sg_status sg_get_layout(sg_grid g, sg_layout* out) {
  SG_CHECK_GRID(g);
  if (!out) return SG_ERR_ARG;
  out->d = g->L.d;
  out->n = g->L.n;
  out->num_points = g->L.N;
  out->num_subspaces = g->L.T;
  out->group_offset = g->L.off;
  out->group_count = g->L.cnt;
  return SG_OK;
}

sg_status sg_destroy(sg_grid g) {
  if (!g) return SG_OK;
  if (g->d_L) {
    DeviceGuard guard(g->device);
    cudaDeviceSynchronize();
    cudaFree(g->d_L);
    if (void* t = g->d_hier_tab.load()) cudaFree(t);
  }
  delete g;
  return SG_OK;
}

sg_status sg_gp2idx(sg_grid g, const int32_t* l, const int32_t* i, uint64_t count, uint64_t* idx) {
  SG_CHECK_GRID(g);
  if (count && (!l || !i || !idx)) return SG_ERR_ARG;
  const int d = g->L.d;
  bool bad = false;
  for (uint64_t q = 0; q < count; ++q) {
    if (valid_point(g->L, l + q * d, i + q * d)) {
      idx[q] = gp2idx(g->L, l + q * d, i + q * d);
    } else {
      idx[q] = UINT64_MAX;
      bad = true;
    }
  }
  if (bad) set_error("sg_gp2idx: some items are not grid points (UINT64_MAX written)");
  return bad ? SG_ERR_RANGE : SG_OK;
}

sg_status sg_idx2gp(sg_grid g, const uint64_t* idx, uint64_t count, int32_t* l, int32_t* i) {
  SG_CHECK_GRID(g);
  if (count && (!l || !i || !idx)) return SG_ERR_ARG;
  const int d = g->L.d;
  bool bad = false;
  for (uint64_t q = 0; q < count; ++q) {
    if (idx[q] < g->L.N) {
      idx2gp(g->L, idx[q], l + q * d, i + q * d);
    } else {
      for (int t = 0; t < d; ++t) l[q * d + t] = i[q * d + t] = -1;
      bad = true;
    }
  }
  if (bad) set_error("sg_idx2gp: some indices are >= N (-1 written)");
  return bad ? SG_ERR_RANGE : SG_OK;
}

sg_status sg_gp2idx_device(sg_grid g, const int32_t* d_l, const int32_t* d_i, uint64_t count, uint64_t* d_idx,
                           void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (count && (!d_l || !d_i || !d_idx)) return SG_ERR_ARG;
  DeviceGuard guard(g->device);
  return launch_gp2idx(g, d_l, d_i, count, d_idx, (cudaStream_t)stream);
}

sg_status sg_idx2gp_device(sg_grid g, const uint64_t* d_idx, uint64_t count, int32_t* d_l, int32_t* d_i,
                           void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (count && (!d_l || !d_i || !d_idx)) return SG_ERR_ARG;
  DeviceGuard guard(g->device);
  return launch_idx2gp(g, d_idx, count, d_l, d_i, (cudaStream_t)stream);
}

sg_status sg_grid_coords_device(sg_grid g, uint64_t first, uint64_t count, void* d_x, sg_dtype dt, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (count && !d_x) return SG_ERR_ARG;
  if (first > g->L.N || count > g->L.N - first) {
    set_error("sg_grid_coords_device: range [%llu, +%llu) exceeds N=%llu", (unsigned long long)first,
              (unsigned long long)count, (unsigned long long)g->L.N);
    return SG_ERR_RANGE;
  }
  DeviceGuard guard(g->device);
  return launch_coords(g, first, count, d_x, dt, (cudaStream_t)stream);
}

sg_status sg_hierarchize(sg_grid g, void* d_values, sg_dtype dt, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (!d_values) return SG_ERR_ARG;
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_hierarchize");
  return launch_hierarchize(g, d_values, dt, (cudaStream_t)stream);
}

sg_status sg_evaluate_workspace_bytes(sg_grid g, uint64_t m, sg_dtype dt, uint32_t flags, size_t* bytes) {
  SG_CHECK_GRID(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (!bytes) return SG_ERR_ARG;
  *bytes = (flags & SG_EVAL_PRESORTED) || m == 0 ? 0 : sfc_workspace_bytes(m);
  return SG_OK;
}

sg_status sg_evaluate(sg_grid g, const void* d_alpha, const void* d_x, uint64_t m, void* d_y, sg_dtype dt,
                      uint32_t flags, void* d_workspace, size_t ws_bytes, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (m == 0) return SG_OK;
  if (!d_alpha || !d_x || !d_y) {
    set_error("sg_evaluate: NULL buffer");
    return SG_ERR_ARG;
  }
  if (m > 0x7fffffffull) {
    set_error("sg_evaluate: at most 2^31-1 queries per call (got %llu)", (unsigned long long)m);
    return SG_ERR_ARG;
  }
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_evaluate");
  cudaStream_t s = (cudaStream_t)stream;
  const uint32_t* perm = nullptr;
  void* own_ws = nullptr;
  sg_status st = SG_OK;
  if (!(flags & SG_EVAL_PRESORTED)) {
    size_t need = sfc_workspace_bytes(m);
    if (!d_workspace) {
      cudaError_t e = cudaMallocAsync(&own_ws, need, s);
      if (e != cudaSuccess) return cuda_fail(e, "sg_evaluate: cudaMallocAsync(workspace)");
      d_workspace = own_ws;
      ws_bytes = need;
    }
    st = launch_sfc_order(g, d_x, m, dt, d_workspace, ws_bytes, nullptr, &perm, s);
  }
  if (st == SG_OK) st = launch_evaluate(g, d_alpha, d_x, perm, m, d_y, dt, flags, s);
  if (own_ws) cudaFreeAsync(own_ws, s);
  return st;
}

sg_status sg_sfc_order(sg_grid g, const void* d_x, uint64_t m, sg_dtype dt, uint32_t* d_perm, void* d_workspace,
                       size_t ws_bytes, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (m == 0) return SG_OK;
  if (!d_x || !d_perm) {
    set_error("sg_sfc_order: NULL buffer");
    return SG_ERR_ARG;
  }
  if (m > 0x7fffffffull) {
    set_error("sg_sfc_order: at most 2^31-1 queries per call (got %llu)", (unsigned long long)m);
    return SG_ERR_ARG;
  }
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_sfc_order");
  cudaStream_t s = (cudaStream_t)stream;
  void* own_ws = nullptr;
  if (!d_workspace) {
    ws_bytes = sfc_workspace_bytes(m);
    cudaError_t e = cudaMallocAsync(&own_ws, ws_bytes, s);
    if (e != cudaSuccess) return cuda_fail(e, "sg_sfc_order: cudaMallocAsync(workspace)");
    d_workspace = own_ws;
  }
  sg_status st = launch_sfc_order(g, d_x, m, dt, d_workspace, ws_bytes, d_perm, nullptr, s);
  if (own_ws) cudaFreeAsync(own_ws, s);
  return st;
}

sg_status sg_evaluate_ordered(sg_grid g, const void* d_alpha, const void* d_x, uint64_t m, const uint32_t* d_perm,
                              uint64_t first, uint64_t count, void* d_y, sg_dtype dt, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (first > m || count > m - first) {
    set_error("sg_evaluate_ordered: range [%llu, +%llu) exceeds m=%llu", (unsigned long long)first,
              (unsigned long long)count, (unsigned long long)m);
    return SG_ERR_RANGE;
  }
  if (count == 0) return SG_OK;
  if (!d_alpha || !d_x || !d_y) {
    set_error("sg_evaluate_ordered: NULL buffer");
    return SG_ERR_ARG;
  }
  if (m > 0x7fffffffull) {
    set_error("sg_evaluate_ordered: at most 2^31-1 queries per batch (got %llu)", (unsigned long long)m);
    return SG_ERR_ARG;
  }
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_evaluate_ordered");
  const size_t es = dtype_size(dt);
  if (d_perm)  // positions first..first+count-1 of the order; x and y indexed by the query's input position
    return launch_evaluate(g, d_alpha, d_x, d_perm + first, count, d_y, dt, SG_EVAL_PRESORTED, (cudaStream_t)stream);
  // no order: the batch is taken as presorted, rows first..first+count-1
  return launch_evaluate(g, d_alpha, (const char*)d_x + first * (size_t)g->L.d * es, nullptr, count,
                         (char*)d_y + first * es, dt, SG_EVAL_PRESORTED, (cudaStream_t)stream);
}

sg_status sg_plane_workspace_bytes(sg_grid g, uint32_t width, uint32_t height, sg_dtype dt, size_t* bytes) {
  SG_CHECK_GRID(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (!bytes) return SG_ERR_ARG;
  *bytes = plane_workspace_bytes(g->L.d, (uint64_t)width * height, dtype_size(dt));
  return SG_OK;
}

sg_status sg_evaluate_plane(sg_grid g, const void* d_alpha, const double* origin, const double* du, const double* dv,
                            uint32_t width, uint32_t height, void* d_image, sg_dtype dt, uint32_t order,
                            void* d_workspace, size_t ws_bytes, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  const uint64_t m = (uint64_t)width * height;
  if (m == 0) return SG_OK;
  if (!d_alpha || !origin || !du || !dv || !d_image) {
    set_error("sg_evaluate_plane: NULL argument");
    return SG_ERR_ARG;
  }
  if (m > 0x7fffffffull || order > 1) {
    set_error("sg_evaluate_plane: need width*height < 2^31 and order 0 or 1");
    return SG_ERR_ARG;
  }
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_evaluate_plane");
  cudaStream_t s = (cudaStream_t)stream;
  const size_t need = plane_workspace_bytes(g->L.d, m, dtype_size(dt));
  void* own = nullptr;
  if (!d_workspace) {
    cudaError_t e = cudaMallocAsync(&own, need, s);
    if (e != cudaSuccess) return cuda_fail(e, "sg_evaluate_plane: cudaMallocAsync(workspace)");
    d_workspace = own;
  } else if (ws_bytes < need) {
    set_error("sg_evaluate_plane: workspace too small (%zu < %zu)", ws_bytes, need);
    return SG_ERR_ARG;
  }
  sg_status st = launch_plane(g, d_alpha, origin, du, dv, width, height, d_image, dt, order, d_workspace, s);
  if (own) cudaFreeAsync(own, s);
  return st;
}

sg_status sg_part_bounds(sg_grid g, uint32_t parts, uint32_t part, uint64_t* first, uint64_t* count) {
  SG_CHECK_GRID(g);
  if (parts == 0 || part >= parts || !first || !count) {
    set_error("sg_part_bounds: need 0 <= part < parts and non-NULL outputs");
    return SG_ERR_ARG;
  }
  PartRange pr;
  part_range(g->L, parts, part, &pr);
  *first = pr.first;
  *count = pr.count;
  return SG_OK;
}

sg_status sg_evaluate_part(sg_grid g, const void* d_alpha_part, uint32_t parts, uint32_t part, const void* d_x,
                           uint64_t m, const uint32_t* d_perm, void* d_y, int accumulate, sg_dtype dt, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (parts == 0 || part >= parts) {
    set_error("sg_evaluate_part: need 0 <= part < parts");
    return SG_ERR_ARG;
  }
  if (m == 0) return SG_OK;
  if (!d_x || !d_y) {
    set_error("sg_evaluate_part: NULL buffer");
    return SG_ERR_ARG;
  }
  if (g->L.d > 12 || g->L.n > 12 || g->L.N >= 0xffffffffull || m > 0x7fffffffull) {
    set_error("sg_evaluate_part: sharded evaluation needs d <= 12, n <= 12, N < 2^32, m < 2^31");
    return SG_ERR_ARG;
  }
  PartRange pr;
  part_range(g->L, parts, part, &pr);
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_evaluate_part");
  cudaStream_t s = (cudaStream_t)stream;
  if (pr.count == 0) {  // an empty part adds nothing; without accumulate y is defined as 0
    if (!accumulate) {
      cudaError_t e = cudaMemsetAsync(d_y, 0, m * dtype_size(dt), s);
      if (e != cudaSuccess) return cuda_fail(e, "sg_evaluate_part: cudaMemsetAsync");
    }
    return SG_OK;
  }
  if (!d_alpha_part) {
    set_error("sg_evaluate_part: NULL surpluses");
    return SG_ERR_ARG;
  }
  GenPart gp = pr.gp;
  gp.accumulate = accumulate ? 1 : 0;
  // the kernel indexes the surpluses with global offsets: hand it the part's base shifted by its first
  // index (only the part's own count values are ever read)
  const void* base = (const char*)d_alpha_part - pr.first * dtype_size(dt);
  ProfScope prof(kProfEval, s);
  bool handled = false;
  const sg_status st = launch_eval_gen(g, base, d_x, d_perm, m, d_y, dt, s, &handled, gp);
  if (st == SG_OK && !handled) {
    set_error("sg_evaluate_part: no generic kernel for d=%d", g->L.d);
    return SG_ERR_ARG;
  }
  return st;
}

sg_status sg_evaluate_host(sg_grid g, const void* d_alpha, const void* h_x, uint64_t m, void* h_y, sg_dtype dt,
                           uint32_t flags, void* stream) {
  SG_CHECK_GRID(g);
  SG_CHECK_DEVICE(g);
  if (!dtype_ok(dt)) return SG_ERR_DTYPE;
  if (m == 0) return SG_OK;
  if (!d_alpha || !h_x || !h_y) return SG_ERR_ARG;
  DeviceGuard guard(g->device);
  NvtxRange nvtx("sg_evaluate_host");
  cudaStream_t s = (cudaStream_t)stream;
  const size_t xb = m * (size_t)g->L.d * dtype_size(dt), yb = m * dtype_size(dt);
  void *dx = nullptr, *dy = nullptr;
  cudaError_t e = cudaMallocAsync(&dx, xb, s);
  if (e != cudaSuccess) return cuda_fail(e, "sg_evaluate_host: cudaMallocAsync");
  e = cudaMallocAsync(&dy, yb, s);
  if (e != cudaSuccess) {
    cudaFreeAsync(dx, s);
    return cuda_fail(e, "sg_evaluate_host: cudaMallocAsync");
  }
  sg_status st = SG_OK;
  e = cudaMemcpyAsync(dx, h_x, xb, cudaMemcpyHostToDevice, s);
  if (e != cudaSuccess) st = cuda_fail(e, "sg_evaluate_host: H2D");
  if (st == SG_OK) st = sg_evaluate(g, d_alpha, dx, m, dy, dt, flags, nullptr, 0, stream);
  if (st == SG_OK) {
    e = cudaMemcpyAsync(h_y, dy, yb, cudaMemcpyDeviceToHost, s);
    if (e != cudaSuccess) st = cuda_fail(e, "sg_evaluate_host: D2H");
  }
  cudaFreeAsync(dx, s);
  cudaFreeAsync(dy, s);
  e = cudaStreamSynchronize(s);
  if (st == SG_OK && e != cudaSuccess) st = cuda_fail(e, "sg_evaluate_host: sync");
  return st;
}

uint64_t sg_kernel_launch_count(void) { return g_launches.load(); }

size_t sg_launched_kernels(char* buf, size_t len) {
  std::string names;
  {
    std::lock_guard<std::mutex> lk(g_kern_mu);
    for (const void* f : g_kernels) {
      const char* nm = nullptr;
      if (cudaFuncGetName(&nm, f) == cudaSuccess && nm) {
        names += nm;
        names += '\n';
      }
    }
  }
  if (buf && len) {
    const size_t k = names.size() < len - 1 ? names.size() : len - 1;
    memcpy(buf, names.data(), k);
    buf[k] = 0;
  }
  return names.size() + 1;
}

sg_status sg_profile_enable(int on) {
  g_prof_on.store(on ? 1 : 0);
  return SG_OK;
}

sg_status sg_profile_read(double* eval_ms, uint64_t* eval_launches, double* hier_ms, uint64_t* hier_launches,
                          int reset) {
  std::lock_guard<std::mutex> lk(g_prof_mu);
  const cudaError_t e = prof_fold(0);
  const sg_status st = e == cudaSuccess ? SG_OK : cuda_fail(e, "sg_profile_read");
  if (eval_ms) *eval_ms = g_prof_ms[kProfEval];
  if (eval_launches) *eval_launches = g_prof_n[kProfEval];
  if (hier_ms) *hier_ms = g_prof_ms[kProfHier];
  if (hier_launches) *hier_launches = g_prof_n[kProfHier];
  if (reset) {
    g_prof_ms[0] = g_prof_ms[1] = 0;
    g_prof_n[0] = g_prof_n[1] = 0;
  }
  return st;
}

const char* sg_status_string(sg_status s) {
  switch (s) {
    case SG_OK: return "SG_OK";
    case SG_ERR_ARG: return "SG_ERR_ARG";
    case SG_ERR_RANGE: return "SG_ERR_RANGE";
    case SG_ERR_OVERFLOW: return "SG_ERR_OVERFLOW";
    case SG_ERR_NOMEM: return "SG_ERR_NOMEM";
    case SG_ERR_CUDA: return "SG_ERR_CUDA";
    case SG_ERR_DTYPE: return "SG_ERR_DTYPE";
    case SG_ERR_NODEV: return "SG_ERR_NODEV";
  }
  return "SG_UNKNOWN";
}

const char* sg_last_error(void) { return t_err; }

const char* sg_build_info(void) { return "libsg sm_100a nvcc " SG_BUILD_FLAGS; }

}  // extern "C"
