// index_kernels.cu -- a8: device-batch gp2idx / idx2gp (Alg. 5, P:L441-L447;
// inverse P:L449) and grid-point coordinates (x_t = i_t / 2^{l_t+1}).
// One thread per item; the layout tables (binmat + index3 offsets) are
// staged once per CTA in shared memory (the paper found binmat in fast on-chip
// memory ~4x faster than recomputing binomials).
#include "common.cuh"

namespace sg {

namespace {

constexpr int kThreads = 256;

__device__ __forceinline__ void stage_layout(const Layout* __restrict__ gL, Layout& sL) {
  const uint32_t* src = reinterpret_cast<const uint32_t*>(gL);
  uint32_t* dst = reinterpret_cast<uint32_t*>(&sL);
  for (int k = threadIdx.x; k < (int)(sizeof(Layout) / 4); k += blockDim.x) dst[k] = src[k];
  __syncthreads();
}

__global__ void __launch_bounds__(kThreads) k_gp2idx(const Layout* __restrict__ gL, const int32_t* __restrict__ l,
                                                     const int32_t* __restrict__ i, uint64_t count,
                                                     uint64_t* __restrict__ idx) {
  __shared__ Layout sL;
  stage_layout(gL, sL);
  const int d = sL.d;
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < count;
       q += (uint64_t)gridDim.x * blockDim.x) {
    int32_t lv[SG_MAX_D], iv[SG_MAX_D];
    for (int t = 0; t < d; ++t) {
      lv[t] = l[q * d + t];
      iv[t] = i[q * d + t];
    }
    idx[q] = valid_point(sL, lv, iv) ? gp2idx(sL, lv, iv) : UINT64_MAX;
  }
}

__global__ void __launch_bounds__(kThreads) k_idx2gp(const Layout* __restrict__ gL, const uint64_t* __restrict__ idx,
                                                     uint64_t count, int32_t* __restrict__ l,
                                                     int32_t* __restrict__ i) {
  __shared__ Layout sL;
  stage_layout(gL, sL);
  const int d = sL.d;
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < count;
       q += (uint64_t)gridDim.x * blockDim.x) {
    int32_t lv[SG_MAX_D], iv[SG_MAX_D];
    uint64_t e = idx[q];
    if (e < sL.N) {
      idx2gp(sL, e, lv, iv);
    } else {
      for (int t = 0; t < d; ++t) lv[t] = iv[t] = -1;
    }
    for (int t = 0; t < d; ++t) {
      l[q * d + t] = lv[t];
      i[q * d + t] = iv[t];
    }
  }
}

template <typename T>
__global__ void __launch_bounds__(kThreads) k_coords(const Layout* __restrict__ gL, uint64_t first, uint64_t count,
                                                     T* __restrict__ x) {
  __shared__ Layout sL;
  stage_layout(gL, sL);
  const int d = sL.d;
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < count;
       q += (uint64_t)gridDim.x * blockDim.x) {
    int32_t lv[SG_MAX_D], iv[SG_MAX_D];
    idx2gp(sL, first + q, lv, iv);
    for (int t = 0; t < d; ++t) x[q * d + t] = (T)ldexp((double)iv[t], -(lv[t] + 1));
  }
}

inline int grid_for(uint64_t count) {
  uint64_t b = (count + kThreads - 1) / kThreads;
  uint64_t cap = (uint64_t)kNumSMs * 16;
  return (int)(b < 1 ? 1 : (b > cap ? cap : b));
}

}  // namespace

sg_status launch_gp2idx(const sg_grid_s* g, const int32_t* l, const int32_t* i, uint64_t count, uint64_t* idx,
                        cudaStream_t s) {
  if (count == 0) return SG_OK;
  k_gp2idx<<<grid_for(count), kThreads, 0, s>>>(g->d_L, l, i, count, idx);
  return launched("k_gp2idx", (const void*)k_gp2idx);
}

sg_status launch_idx2gp(const sg_grid_s* g, const uint64_t* idx, uint64_t count, int32_t* l, int32_t* i,
                        cudaStream_t s) {
  if (count == 0) return SG_OK;
  k_idx2gp<<<grid_for(count), kThreads, 0, s>>>(g->d_L, idx, count, l, i);
  return launched("k_idx2gp", (const void*)k_idx2gp);
}

sg_status launch_coords(const sg_grid_s* g, uint64_t first, uint64_t count, void* x, sg_dtype dt, cudaStream_t s) {
  if (count == 0) return SG_OK;
  if (dt == SG_F64)
    k_coords<double><<<grid_for(count), kThreads, 0, s>>>(g->d_L, first, count, (double*)x);
  else
    k_coords<float><<<grid_for(count), kThreads, 0, s>>>(g->d_L, first, count, (float*)x);
  return launched("k_coords", dt == SG_F64 ? (const void*)k_coords<double> : (const void*)k_coords<float>);
}

}  // namespace sg
