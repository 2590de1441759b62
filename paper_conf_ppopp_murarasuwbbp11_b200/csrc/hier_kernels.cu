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

template <typename T>
__global__ void __launch_bounds__(kThreads) k_hier_family(const Layout* __restrict__ gL, int t, T* __restrict__ v) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* fam = reinterpret_cast<T*>(smem_raw);
  __shared__ FamilyInfo fi;
  __shared__ Layout sL;
  {
    const uint32_t* src = reinterpret_cast<const uint32_t*>(gL);
    uint32_t* dst = reinterpret_cast<uint32_t*>(&sL);
    for (int k = threadIdx.x; k < (int)(sizeof(Layout) / 4); k += blockDim.x) dst[k] = src[k];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int32_t lv[SG_MAX_D];
    family_levels(sL, t, blockIdx.x, lv);
    int s = 0, suf = 0;
    for (int u = 0; u < sL.d; ++u) {
      s += lv[u];
      if (u > t) suf += lv[u];
    }
    fi.s = s;
    fi.suf = suf;
    fi.L = sL.n - s;
    for (int k = 0; k < fi.L; ++k) {
      lv[t] = k;
      int j = s + k;
      fi.base[k] = sL.off[j] + (subspace_rank(sL, lv) << j);
    }
  }
  __syncthreads();
  const int s = fi.s, L = fi.L, suf = fi.suf;
  const uint32_t E = ((1u << L) - 1u) << s;  // family size 2^s (2^L - 1)
  // load: element e lies in block k = floor(log2((e >> s) + 1))
  for (uint32_t e = threadIdx.x; e < E; e += blockDim.x) {
    int k = 31 - __clz((e >> s) + 1);
    uint32_t w = e - (((1u << k) - 1u) << s);
    fam[e] = v[fi.base[k] + w];
  }
  __syncthreads();
  const uint32_t lomask = (1u << suf) - 1u;
  for (uint32_t e = (1u << s) + threadIdx.x; e < E; e += blockDim.x) {  // blocks k >= 1
    int k = 31 - __clz((e >> s) + 1);
    uint32_t w = e - (((1u << k) - 1u) << s);
    uint32_t lo = w & lomask;
    uint32_t c = (w >> suf) & ((1u << k) - 1u);
    uint32_t hi = w >> (suf + k);
    T vl = T(0), vr = T(0);
    if (c != 0) {  // left parent at c / 2^k
      int b = __ffs(c) - 1;
      int kp = k - 1 - b;
      uint32_t cp = (c >> b) >> 1;
      vl = fam[(((1u << kp) - 1u) << s) + ((((hi << kp) + cp) << suf) | lo)];
    }
    if (c + 1 != (1u << k)) {  // right parent at (c+1) / 2^k
      int b = __ffs(c + 1) - 1;
      int kp = k - 1 - b;
      uint32_t cp = ((c + 1) >> b) >> 1;
      vr = fam[(((1u << kp) - 1u) << s) + ((((hi << kp) + cp) << suf) | lo)];
    }
    v[fi.base[k] + w] = fam[e] - (vl + vr) / T(2);
  }
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
    cudaError_t e = cudaFuncSetAttribute(k_hier_family<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)fam_bytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(k_hier_family)");
    // families with |l_{-t}| <= n-2: sum_{s<=n-2} C(s+d-2, d-2) = C(n-2+d-1, d-1)
    uint64_t F = (d == 1) ? 1 : L.C(d - 1, n - 2);
    if (F > 0x7fffffffull) return SG_ERR_OVERFLOW;
    for (int t = 0; t < d; ++t) {
      k_hier_family<T><<<(unsigned)F, kThreads, fam_bytes, s>>>(g->d_L, t, v);
      sg_status st = launched("k_hier_family");
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
    sg_status st = launched("k_hier_global");
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
