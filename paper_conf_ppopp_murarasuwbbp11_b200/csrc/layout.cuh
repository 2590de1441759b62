// layout.cuh -- B0 layout core of libsg: the compact sparse-grid layout of
// Murarasu et al. PPoPP'11 Sec. 4, as __host__ __device__
// inline functions over a POD table.  Independent of oracle/ (shares no code).
//
//   idx(l, i) = off[|l|] + rank(l) * 2^{|l|} + index1(l, i)
//   off[j]    = sum_{s<j} C(d-1+s, d-1) 2^s
//   rank(l)   = sum_{t=1}^{d-1} C(t+S_t, t) - C(t+S_{t-1}, t),
//               S_t = l_0 + ... + l_t                              (eq. 4)
//   index1    = digits (i_t-1)/2 in mixed radix 2^{l_t}, dim 0 most
//               significant                                        (Alg 5 l.1-4)
#pragma once
#include <stdint.h>

#include "../../include/sg.h"

#ifdef __CUDACC__
#define SG_HD __host__ __device__ __forceinline__
#else
#define SG_HD inline
#endif

namespace sg {

// binom(t, s) = C(t + s, t): the paper's "binmat", rows t = 0..SG_MAX_D,
// columns s = 0..SG_MAX_N.  C(64, 32) < 2^64, so every entry is exact.
constexpr int kBinRows = SG_MAX_D + 1;
constexpr int kBinCols = SG_MAX_N + 1;

struct Layout {
  int32_t d, n;
  uint64_t N;                  // number of points
  uint64_t T;                  // number of subspaces = terms per evaluation
  uint64_t off[SG_MAX_N + 1];  // group offsets index3(j), off[n] = N
  uint64_t cnt[SG_MAX_N];      // subspaces per group C(d-1+j, d-1)
  uint64_t bin[kBinRows][kBinCols];

  SG_HD uint64_t C(int t, int s) const { return bin[t][s]; }  // C(t+s, t)
};

// Fill the tables; returns false on overflow (N >= 2^62).
inline bool build_layout(int d, int n, Layout* L) {
  L->d = d;
  L->n = n;
  for (int t = 0; t < kBinRows; ++t) {
    for (int s = 0; s < kBinCols; ++s) {
      if (t == 0 || s == 0) L->bin[t][s] = 1;
      else L->bin[t][s] = L->bin[t - 1][s] + L->bin[t][s - 1];  // C(t+s,t) = C(t+s-1,t-1) + C(t+s-1,t)
    }
  }
  uint64_t acc = 0, subs = 0;
  for (int j = 0; j <= SG_MAX_N; ++j) L->off[j] = 0;
  for (int j = 0; j < n; ++j) {
    L->off[j] = acc;
    uint64_t c = L->bin[d - 1][j];
    L->cnt[j] = c;
    subs += c;
    if (c > (((uint64_t)1 << 62) >> j)) return false;
    acc += c << j;
    if (acc >= ((uint64_t)1 << 62)) return false;
  }
  L->off[n] = acc;
  L->N = acc;
  L->T = subs;
  return true;
}

// rank of level vector l within its group, eq. (4)
SG_HD uint64_t subspace_rank(const Layout& L, const int32_t* l) {
  int S = l[0];
  uint64_t r = 0;
  for (int t = 1; t < L.d; ++t) {
    int S2 = S + l[t];
    r += L.C(t, S2) - L.C(t, S);
    S = S2;
  }
  return r;
}

// true iff (l, i) is a point of the grid
SG_HD bool valid_point(const Layout& L, const int32_t* l, const int32_t* i) {
  int s = 0;
  for (int t = 0; t < L.d; ++t) {
    if (l[t] < 0 || l[t] > L.n - 1) return false;
    s += l[t];
    if ((i[t] & 1) == 0 || i[t] < 1 || (int64_t)i[t] > (((int64_t)2 << l[t]) - 1)) return false;
  }
  return s <= L.n - 1;
}

// gp2idx; caller checks valid_point first
SG_HD uint64_t gp2idx(const Layout& L, const int32_t* l, const int32_t* i) {
  uint64_t index1 = 0;
  int j = 0;
  for (int t = 0; t < L.d; ++t) {
    index1 = (index1 << l[t]) | (uint64_t)(i[t] >> 1);
    j += l[t];
  }
  return L.off[j] + (subspace_rank(L, l) << j) + index1;
}

// idx2gp; caller checks idx < N
SG_HD void idx2gp(const Layout& L, uint64_t idx, int32_t* l, int32_t* i) {
  int j = L.n - 1;
  while (L.off[j] > idx) --j;  // group: off[j] <= idx < off[j+1]
  uint64_t r = idx - L.off[j];
  uint64_t rank = r >> j;
  uint64_t index1 = r & ((((uint64_t)1) << j) - 1);
  // unrank in Alg. 3 order: component t = d-1 .. 1, each block with l_t = k holds
  // |L^t_{m-k}| = C(t-1+m-k, t-1) vectors
  int m = j;
  for (int t = L.d - 1; t >= 1; --t) {
    int k = 0;
    while (true) {
      uint64_t c = L.C(t - 1, m - k);
      if (rank < c) break;
      rank -= c;
      ++k;
    }
    l[t] = k;
    m -= k;
  }
  l[0] = m;
  for (int t = L.d - 1; t >= 0; --t) {
    uint64_t k = index1 & ((((uint64_t)1) << l[t]) - 1);
    index1 >>= l[t];
    i[t] = (int32_t)(2 * k + 1);
  }
}

}  // namespace sg
