// sfc_kernels.cu -- a1: order a query batch along a Morton (Z-order) curve.
//
// The paper blocks evaluation points so that a subspace brought into cache
// serves many evaluations and copies coords coalesced to shared
// memory.  On B200 the equivalent is spatial locality *within a
// warp and a CTA*: queries that are close in space fall into the same cells
// of the coarse subspaces, so their surplus gathers coalesce into few L1/L2
// sectors.  Keys: b = min(20, 63/d) bits per dimension, interleaved with the
// most significant bit of every dimension first; CUB radix sort of
// (key, query index) pairs on the caller's stream.
#include <cub/device/device_radix_sort.cuh>

#include <stdlib.h>

#include "common.cuh"

namespace sg {

namespace {

constexpr int kThreads = 256;

inline int morton_bits(int d) {
  int b = 63 / d;
  return b > 20 ? 20 : (b < 1 ? 1 : b);
}

// Plane lag of dimension t.  In the layout the in-subspace index has
// dimension 0 as its most significant digit and dimension d-1 as its fastest
// one (Alg. 5), and a warp's fp64 gather costs, per half-warp, the
// largest number of distinct words that fall into one L1 bank pair (address
// bits 3-6, i.e. the low 4 bits of the index; profiles/r01_ubench_l1_gather.txt).
// Queries of a warp that differ in the high dimensions (coarse digits) but
// agree in the low ones land in the same bank pair and serialise; queries that
// differ in the fast dimensions do not.  Entering the fast dimensions later
// in the curve makes warps compact in dimensions 0..d/2 and elongated in the
// fast ones: at d = 10 this cuts the modelled L1 cycles per gather from 4.11
// to 3.27 (SURVEY-style simulation over 10^7 uniform points, groups 5-10).
__host__ __device__ inline int morton_lag(int t, int start, int cap) {
  const int lag = t - start;  // start = d / 2 (d >= 4), d (no lag) below
  return lag <= 0 ? 0 : (lag < cap ? lag : cap);
}

template <typename T>
__global__ void __launch_bounds__(kThreads) k_morton(const T* __restrict__ x, uint64_t m, int d, int bits, int cap, int start,
                                                     uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < m; q += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t c[SG_MAX_D];
    const double scale = (double)(1u << bits);
    const double top = scale - 1.0;
    for (int t = 0; t < d; ++t) {
      double v = floor((double)x[q * d + t] * scale);
      v = v >= 0.0 ? v : 0.0;  // also maps NaN to 0
      v = v <= top ? v : top;
      c[t] = (uint32_t)v;
    }
    // bit planes from the most significant one; dimension t enters lag(t)
    // planes late (see morton_lag), so every dimension keeps `bits` bits
    uint64_t key = 0;
    const int lmax = morton_lag(d - 1, start, cap);
    for (int p = 0; p < bits + lmax; ++p)
      for (int t = 0; t < d; ++t) {
        const int b = p - morton_lag(t, start, cap);  // bit of dimension t, 0 = its MSB
        if (b >= 0 && b < bits) key = (key << 1) | ((c[t] >> (bits - 1 - b)) & 1u);
      }
    keys[q] = key;
    vals[q] = (uint32_t)q;
  }
}

inline size_t align_up(size_t v) { return (v + 255) & ~(size_t)255; }

size_t cub_temp_bytes(uint64_t m) {
  size_t temp = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, temp, (const uint64_t*)nullptr, (uint64_t*)nullptr,
                                  (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)m, 0, 64);
  return temp;
}

}  // namespace

size_t sfc_workspace_bytes(uint64_t m) {
  return 2 * align_up(m * sizeof(uint64_t)) + 2 * align_up(m * sizeof(uint32_t)) + align_up(cub_temp_bytes(m));
}

sg_status launch_sfc_order(const sg_grid_s* g, const void* x, uint64_t m, sg_dtype dt, void* ws, size_t ws_bytes,
                           uint32_t* perm_dst, const uint32_t** perm_out, cudaStream_t s) {
  if (m > 0x7fffffffull) {
    set_error("sg_evaluate: m = %llu exceeds 2^31-1 queries per call", (unsigned long long)m);
    return SG_ERR_ARG;
  }
  if (ws_bytes < sfc_workspace_bytes(m)) {
    set_error("sg_evaluate: workspace too small (%zu < %zu)", ws_bytes, sfc_workspace_bytes(m));
    return SG_ERR_ARG;
  }
  char* p = (char*)ws;
  uint64_t* k0 = (uint64_t*)p;
  p += align_up(m * 8);
  uint64_t* k1 = (uint64_t*)p;
  p += align_up(m * 8);
  uint32_t* v0 = (uint32_t*)p;
  p += align_up(m * 4);
  uint32_t* v1 = (uint32_t*)p;
  p += align_up(m * 4);
  size_t temp = cub_temp_bytes(m);
  const int d = g->L.d, bits = morton_bits(d);
  // lag cap 2 (dimensions 7, 8, 9 of 10 one, two, two planes late): measured best at cfg3 once the
  // evaluation kernel is closer to its memory ceiling (r02: 7.83e6 evals/s at caps 2-4 vs 7.62e6 at cap 1,
  // profiles/r02_split.txt; the L1 bank-pair model, gives 3.90 vs 4.57 cycles per group-10
  // gather); r01's cap 1 was best for the latency-bound v7 kernel (profiles/r01_v5_variants.txt)
  int cap = bits / 2 < 2 ? bits / 2 : 2;
#ifdef SG_EXP  // experiment builds only (libsg_exp.so): curve shape from the environment
  if (const char* e = getenv("SG_EXP_LAGCAP")) cap = atoi(e);
#endif
  // lag(t) = min(cap, t - start) for t > start; start = d / 2 + 1: measured best at cfg3 (d = 10: dimensions
  // 7-9 one plane late, 7.08e6 evals/s vs 6.88 / 6.97 / 6.99-7.01 / 7.01e6 at start 3 / 4 / 5 / 7,
  // profiles/r01_v5_variants.txt)
  int start = d < 4 ? d : d / 2 + 1;
#ifdef SG_EXP
  if (const char* e = getenv("SG_EXP_LAGSTART")) start = atoi(e);
#endif
  uint64_t blocks = (m + kThreads - 1) / kThreads;
  if (blocks > (uint64_t)kNumSMs * 32) blocks = (uint64_t)kNumSMs * 32;
  if (dt == SG_F64)
    k_morton<double><<<(unsigned)blocks, kThreads, 0, s>>>((const double*)x, m, d, bits, cap, start, k0, v0);
  else
    k_morton<float><<<(unsigned)blocks, kThreads, 0, s>>>((const float*)x, m, d, bits, cap, start, k0, v0);
  sg_status st = launched("k_morton", dt == SG_F64 ? (const void*)k_morton<double> : (const void*)k_morton<float>);
  if (st != SG_OK) return st;
  // the sort is deterministic (stable LSD radix sort of (key, index) pairs): every rank that orders the same
  // batch gets the same permutation (ranks agree on one global order without communicating)
  uint32_t* vout = perm_dst ? perm_dst : v1;
  cudaError_t e = cub::DeviceRadixSort::SortPairs(p, temp, k0, k1, v0, vout, (int)m, 0, d * bits, s);
  if (e != cudaSuccess) return cuda_fail(e, "cub::DeviceRadixSort::SortPairs");
  if (perm_out) *perm_out = vout;
  return SG_OK;
}

}  // namespace sg
