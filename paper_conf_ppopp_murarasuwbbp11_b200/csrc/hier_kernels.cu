// hier_kernels.cu -- a7: hierarchization (compression), Sec. 3.1 / 4.3.
//
// Semantics (Alg. 1; multi-d sweep; Alg. 6): for
// t = 0..d-1, every point (l, i) with l_t >= 1 becomes
//     v <- v - (v_left + v_right) / 2
// where v_left / v_right are the values (after pass t-1) of its 1D
// hierarchical parents along t, at x_t -/+ 2^-(l_t+1), and 0 on the boundary.
//
// Schedule (new; the paper launched one kernel per level group with one CTA
// per subspace and a CPU barrier between groups): a *pole family* for
// dimension t is the set of subspaces sharing l_{-t} (all levels except l_t).
// Its L = n - |l_{-t}| subspaces are each one contiguous block of 2^{|l|}
// values, 2^n - 2^{|l_{-t}|} values in total, and every 1D pole
// along t -- and therefore every parent a point needs -- lies inside it.  One
// CTA loads a family into shared memory with coalesced reads, computes every
// new value from the pass-(t-1) values, and writes the changed points back:
// one launch per dimension is the only barrier (reading G11).  Families with
// L = 1 contain only l_t = 0 points, which never change, and are skipped.
#include "common.cuh"

namespace sg {

namespace {

constexpr int kThreads = 256;

struct FamilyInfo {
  uint64_t base[SG_MAX_N];  // global offset of the block with l_t = k
  int s, L, suf;            // |l_{-t}|, number of blocks, sum_{u>t} l_u
};

// Unrank family f of dimension t: (d-1)-dim level vectors with sum <= n-2,
// ordered by sum, then in Alg. 3 order.  Fills `lv` (d entries, lv[t] = 0).
__device__ bool family_levels(const Layout& L, int t, uint64_t f, int32_t* lv) {
  const int d = L.d, n = L.n;
  const int dm = d - 1;  // dimensions of l_{-t}
  int s = 0;
  for (;; ++s) {
    if (s > n - 2) return false;
    uint64_t c = dm == 0 ? (s == 0 ? 1 : 0) : L.C(dm - 1, s);  // |L^{d-1}_s|
    if (f < c) break;
    f -= c;
  }
  int32_t w[SG_MAX_D];
  int m = s;
  for (int u = dm - 1; u >= 1; --u) {
    int k = 0;
    while (true) {
      uint64_t c = L.C(u - 1, m - k);
      if (f < c) break;
      f -= c;
      ++k;
    }
    w[u] = k;
    m -= k;
  }
  if (dm >= 1) w[0] = m;
  for (int u = 0, v = 0; u < d; ++u) lv[u] = (u == t) ? 0 : w[v++];
  return true;
}

// ---- v2: family tables built once per grid (first call), so a family's CTA
// needs no serial set-up (v1: thread 0 unranked the family and ranked its L
// blocks while 255 threads waited at a barrier, after copying the 8.6 KB
// Layout into shared memory -- 47% barrier stalls, profiles/r01_v3_hier_ncu.txt).
//
// Per dimension t and family f: info[2f] = |l_{-t}| | (sum_{u>t} l_u) << 8,
// info[2f+1] = index of the family's first block base in `base`, and
// base[first + k] = global offset of the family's block with l_t = k.
// One CTA per family loads the family into shared memory (block by block,
// coalesced), then computes every l_t >= 1 point from its two 1D parents
// (Alg. 1 / Alg. 6) and writes it back.
struct HierTab {
  uint64_t F;          // families per dimension (|l_{-t}| <= n-2)
  uint64_t nbase;      // block bases per dimension (= number of subspaces with |l_{-t}| <= n-2)
  uint32_t* info;      // [d][F][2]
  uint64_t* base;      // [d][nbase]
};

template <int DUMMY = 0>
__global__ void __launch_bounds__(kThreads) k_hier_table(const Layout* __restrict__ gL, int t, uint64_t F,
                                                         uint32_t* __restrict__ info, uint64_t* __restrict__ base) {
  const Layout& L = *gL;
  const uint64_t f = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (f >= F) return;
  int32_t lv[SG_MAX_D];
  family_levels(L, t, f, lv);
  int s = 0, suf = 0;
  for (int u = 0; u < L.d; ++u) {
    s += lv[u];
    if (u > t) suf += lv[u];
  }
  // first = sum over the families before f of their block counts n - s':
  // families are ordered by s' (|L^{d-1}_{s'}| = C(s'+d-2, d-2) of them), then in Alg. 3 order
  const int dm = L.d - 1;
  uint64_t first = 0, before = 0;
  for (int sp = 0; sp < s; ++sp) {
    const uint64_t c = dm == 0 ? (sp == 0 ? 1 : 0) : L.C(dm - 1, sp);
    first += c * (uint64_t)(L.n - sp);
    before += c;
  }
  first += (f - before) * (uint64_t)(L.n - s);
  info[2 * f] = (uint32_t)s | ((uint32_t)suf << 8);
  info[2 * f + 1] = (uint32_t)first;
  for (int k = 0; k < L.n - s; ++k) {
    lv[t] = k;
    const int j = s + k;
    base[first + k] = L.off[j] + (subspace_rank(L, lv) << j);
  }
}

template <typename T>
__global__ void __launch_bounds__(kThreads) k_hier_family2(int n, const uint32_t* __restrict__ info,
                                                           const uint64_t* __restrict__ bases, T* __restrict__ v) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* fam = reinterpret_cast<T*>(smem_raw);
  __shared__ uint64_t base[SG_MAX_N];
  const uint32_t w0 = __ldg(info + 2 * blockIdx.x), first = __ldg(info + 2 * blockIdx.x + 1);
  const int s = (int)(w0 & 0xff), suf = (int)(w0 >> 8), L = n - s;
  if ((int)threadIdx.x < L) base[threadIdx.x] = __ldg(bases + first + threadIdx.x);
  __syncthreads();
  const uint32_t E = ((1u << L) - 1u) << s;  // family size 2^s (2^L - 1)
  // Flat index w over the family: block k holds 2^(s+k) consecutive values at w = 2^(s+k) - 2^s
  // (shared-memory offset = w), i.e. k = floor(log2(w + 2^s)) - s.  v3: every thread first issues
  // all its loads of the family (independent, one round trip), then stores them to shared memory;
  // v2 loaded block by block (one round trip per block: latency-bound, long_scoreboard 58%,
  // profiles/r01_v7_hier_ncu.txt).
  constexpr int U = 8;
  const uint32_t two_s = 1u << s;
  for (uint32_t w0 = 0; w0 < E; w0 += U * blockDim.x) {
    T val[U];
#pragma unroll
    for (int i = 0; i < U; ++i) {
      const uint32_t w = w0 + i * blockDim.x + threadIdx.x;
      if (w < E) {
        const uint32_t p = w + two_s;
        const int k = 31 - __clz(p) - s;
        val[i] = v[base[k] + (p - (1u << (s + k)))];
      }
    }
#pragma unroll
    for (int i = 0; i < U; ++i) {
      const uint32_t w = w0 + i * blockDim.x + threadIdx.x;
      if (w < E) fam[w] = val[i];
    }
  }
  __syncthreads();
  // every point of blocks k >= 1 from its two 1D parents (blocks < k), written straight to global
  const uint32_t lomask = (1u << suf) - 1u;
  for (uint32_t w = two_s + threadIdx.x; w < E; w += blockDim.x) {
    const uint32_t p = w + two_s;
    const int k = 31 - __clz(p) - s;
    const uint32_t wl = p - (1u << (s + k));  // index inside block k
    const uint32_t lo = wl & lomask;
    const uint32_t c = (wl >> suf) & ((1u << k) - 1u);
    const uint32_t hi = wl >> (suf + k);
    T vl = T(0), vr = T(0);
    if (c != 0) {  // left parent at c / 2^k
      const int b = __ffs(c) - 1;
      const int kp = k - 1 - b;
      const uint32_t cp = (c >> b) >> 1;
      vl = fam[(((1u << kp) - 1u) << s) + ((((hi << kp) + cp) << suf) | lo)];
    }
    if (c + 1 != (1u << k)) {  // right parent at (c+1) / 2^k
      const int b = __ffs(c + 1) - 1;
      const int kp = k - 1 - b;
      const uint32_t cp = ((c + 1) >> b) >> 1;
      vr = fam[(((1u << kp) - 1u) << s) + ((((hi << kp) + cp) << suf) | lo)];
    }
    v[base[k] + wl] = fam[w] - (vl + vr) / T(2);
  }
}

sg_status hier_table(const sg_grid_s* g, HierTab* tab) {
  const Layout& L = g->L;
  const int d = L.d, n = L.n;
  tab->F = (d == 1) ? 1 : L.C(d - 1, n - 2);
  // block bases per dimension: sum over families of n - |l_{-t}|
  uint64_t nb = 0;
  for (int sp = 0; sp <= n - 2; ++sp) nb += (d == 1 ? (sp == 0 ? 1 : 0) : L.C(d - 2, sp)) * (uint64_t)(n - sp);
  tab->nbase = nb;
  void* tabs = g->d_hier_tab.load(std::memory_order_acquire);
  if (!tabs) {
    std::lock_guard<std::mutex> lk(g->hier_mu);
    tabs = g->d_hier_tab.load(std::memory_order_acquire);
    if (!tabs) {
      // built on a private stream and synchronised before publishing: a later
      // call on any other stream must never see half-written tables
      const size_t bytes = (size_t)d * (tab->F * 2 * sizeof(uint32_t) + nb * sizeof(uint64_t));
      cudaStream_t bs;
      cudaError_t e = cudaStreamCreateWithFlags(&bs, cudaStreamNonBlocking);
      if (e != cudaSuccess) return cuda_fail(e, "cudaStreamCreate(hierarchization tables)");
      e = cudaMalloc(&tabs, bytes);
      if (e != cudaSuccess) {
        cudaStreamDestroy(bs);
        return cuda_fail(e, "cudaMalloc(hierarchization tables)");
      }
      uint64_t* b = (uint64_t*)tabs;
      uint32_t* in = (uint32_t*)(b + (size_t)d * nb);
      sg_status st = SG_OK;
      for (int t = 0; t < d && st == SG_OK; ++t) {
        const unsigned blocks = (unsigned)((tab->F + kThreads - 1) / kThreads);
        k_hier_table<<<blocks, kThreads, 0, bs>>>(g->d_L, t, tab->F, in + (size_t)t * tab->F * 2, b + (size_t)t * nb);
        st = launched("k_hier_table", (const void*)k_hier_table<0>);
      }
      e = cudaStreamSynchronize(bs);
      cudaStreamDestroy(bs);
      if (st == SG_OK && e != cudaSuccess) st = cuda_fail(e, "cudaStreamSynchronize(hierarchization tables)");
      if (st != SG_OK) {
        cudaFree(tabs);
        return st;
      }
      g->d_hier_tab.store(tabs, std::memory_order_release);
    }
  }
  tab->base = (uint64_t*)tabs;
  tab->info = (uint32_t*)(tab->base + (size_t)d * nb);
  return SG_OK;
}

// Fallback for families larger than shared memory: one thread per point,
// parents read from the previous pass' buffer (ping-pong, out of place).
template <typename T>
__global__ void __launch_bounds__(kThreads) k_hier_global(const Layout* __restrict__ gL, int t,
                                                          const T* __restrict__ in, T* __restrict__ out) {
  __shared__ Layout sL;
  {
    const uint32_t* src = reinterpret_cast<const uint32_t*>(gL);
    uint32_t* dst = reinterpret_cast<uint32_t*>(&sL);
    for (int k = threadIdx.x; k < (int)(sizeof(Layout) / 4); k += blockDim.x) dst[k] = src[k];
  }
  __syncthreads();
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < sL.N; e += (uint64_t)gridDim.x * blockDim.x) {
    int32_t lv[SG_MAX_D], iv[SG_MAX_D];
    idx2gp(sL, e, lv, iv);
    T val = in[e];
    if (lv[t] > 0) {
      const int lt = lv[t], it = iv[t];
      T vl = T(0), vr = T(0);
      if (it - 1 != 0) {
        int b = __ffs(it - 1) - 1;
        lv[t] = lt - b;
        iv[t] = (it - 1) >> b;
        vl = in[gp2idx(sL, lv, iv)];
      }
      if (it + 1 != (2 << lt)) {
        int b = __ffs(it + 1) - 1;
        lv[t] = lt - b;
        iv[t] = (it + 1) >> b;
        vr = in[gp2idx(sL, lv, iv)];
      }
      val = val - (vl + vr) / T(2);
    }
    out[e] = val;
  }
}

template <typename T>
sg_status hierarchize_t(const sg_grid_s* g, T* v, cudaStream_t s) {
  const Layout& L = g->L;
  const int d = L.d, n = L.n;
  if (n < 2) return SG_OK;  // only the level-0 point: its surplus is its value
  const size_t fam_bytes = (((size_t)1 << n) - 1) * sizeof(T);
  int dev = 0, max_smem = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const size_t static_smem = sizeof(Layout) + sizeof(FamilyInfo) + 64;
  if (fam_bytes + static_smem <= (size_t)max_smem) {
    HierTab tab;
    sg_status st = hier_table(g, &tab);
    if (st != SG_OK) return st;
    // the family size differs per grid: opt in to the device maximum once (a permission only; the
    // launch's own dynamic size decides occupancy)
    static std::atomic<uint64_t> attr_done{0};
    st = set_smem_attr(k_hier_family2<T>, attr_done, (size_t)max_smem - static_smem, -1,
                       "cudaFuncSetAttribute(k_hier_family2)");
    if (st != SG_OK) return st;
    if (tab.F > 0x7fffffffull) return SG_ERR_OVERFLOW;
    for (int t = 0; t < d; ++t) {
      k_hier_family2<T><<<(unsigned)tab.F, kThreads, fam_bytes, s>>>(n, tab.info + (size_t)t * tab.F * 2,
                                                                       tab.base + (size_t)t * tab.nbase, v);
      st = launched("k_hier_family2", (const void*)k_hier_family2<T>);
      if (st != SG_OK) return st;
    }
    return SG_OK;
  }
  // large grids: ping-pong through a scratch buffer
  T* tmp = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&tmp, L.N * sizeof(T), s);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMallocAsync(hierarchize scratch)");
  uint64_t blocks = (L.N + kThreads - 1) / kThreads;
  if (blocks > (uint64_t)kNumSMs * 32) blocks = (uint64_t)kNumSMs * 32;
  T* a = v;
  T* b = tmp;
  for (int t = 0; t < d; ++t) {
    k_hier_global<T><<<(unsigned)blocks, kThreads, 0, s>>>(g->d_L, t, a, b);
    sg_status st = launched("k_hier_global", (const void*)k_hier_global<T>);
    if (st != SG_OK) return st;
    T* c = a;
    a = b;
    b = c;
  }
  if (a != v) {
    e = cudaMemcpyAsync(v, a, L.N * sizeof(T), cudaMemcpyDeviceToDevice, s);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync(hierarchize)");
  }
  e = cudaFreeAsync(tmp, s);
  return e == cudaSuccess ? SG_OK : cuda_fail(e, "cudaFreeAsync");
}

}  // namespace

sg_status launch_hierarchize(const sg_grid_s* g, void* v, sg_dtype dt, cudaStream_t s) {
  ProfScope prof(kProfHier, s);
  if (dt == SG_F64) return hierarchize_t<double>(g, (double*)v, s);
  return hierarchize_t<float>(g, (float*)v, s);
}

}  // namespace sg
