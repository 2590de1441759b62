// bankpair.c -- CPU model of the L1 data-stage cost of the evaluation gathers:
// a warp-wide LDG.64 costs, per 16-lane half, the largest number of distinct 8-byte words that
// fall into one bank pair (address bits 3-6), measured in profiles/r01_ubench_l1_gather.txt.
// Queries: the cfg3 SplitMix64 stream (sginputs); order: a sort key (variants below); cost averaged
// over sampled warps and sampled subspaces of each level group, weighted by terms.
//   gcc -O3 -fopenmp -o /tmp/bp scripts/sim/bankpair.c -lm && /tmp/bp M ORDER [params]
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define D 10
#define NM 11
static uint64_t sm64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
typedef struct { uint64_t key; uint32_t q; } KV;
static int cmpkv(const void* a, const void* b) {
  const KV* x = a; const KV* y = b;
  return x->key < y->key ? -1 : x->key > y->key ? 1 : (x->q < y->q ? -1 : x->q > y->q);
}
static int lagf(int t, int start, int cap) { int l = t - start; return l <= 0 ? 0 : (l < cap ? l : cap); }

int main(int argc, char** argv) {
  const uint64_t m = argc > 1 ? strtoull(argv[1], 0, 10) : 10000000;
  const int order = argc > 2 ? atoi(argv[2]) : 1;
  const int start = argc > 3 ? atoi(argv[3]) : 6, cap = argc > 4 ? atoi(argv[4]) : 1;
  const int nwarps = argc > 5 ? atoi(argv[5]) : 400, nsub = argc > 6 ? atoi(argv[6]) : 3000;
  const uint64_t seed = 0x5EED0003ull;
  uint16_t* K = malloc(m * D * sizeof(uint16_t));
  KV* kv = malloc(m * sizeof(KV));
  const int bits = 63 / D;  // 6
#pragma omp parallel for
  for (uint64_t q = 0; q < m; ++q) {
    uint32_t c[D];
    for (int t = 0; t < D; ++t) {
      double x = ((double)(sm64((q * D + t) ^ seed) >> 11) + 0.5) * 0x1p-53;
      K[q * D + t] = (uint16_t)floor(x * 1024.0);
      c[t] = (uint32_t)floor(x * (double)(1u << bits));
    }
    uint64_t key = 0;
    if (order == 0) {  // input order
      key = q;
    } else if (order == 1) {  // Morton with plane lags (start, cap)
      int lmax = lagf(D - 1, start, cap);
      for (int p = 0; p < bits + lmax; ++p)
        for (int t = 0; t < D; ++t) {
          int b = p - lagf(t, start, cap);
          if (b >= 0 && b < bits) key = (key << 1) | ((c[t] >> (bits - 1 - b)) & 1u);
        }
    } else if (order == 2) {  // Morton, dimensions interleaved in reverse (dim 9 first in each plane)
      for (int p = 0; p < bits; ++p)
        for (int t = D - 1; t >= 0; --t) key = (key << 1) | ((c[t] >> (bits - 1 - p)) & 1u);
    }
    kv[q].key = key;
    kv[q].q = (uint32_t)q;
  }
  if (order != 0) qsort(kv, m, sizeof(KV), cmpkv);
  // level vectors per group in Alg. 3 order (l_{D-1} slowest), sampled
  double tot_cost = 0, tot_terms = 0, tot_sect = 0, tot_lines = 0;
  uint64_t rs = 12345;
  for (int j = 0; j < NM; ++j) {
    // enumerate all compositions of j into D parts (count C(j+9,9))
    int cntj = 0, cap_l = 200000;
    int (*L)[D] = malloc(sizeof(int[D]) * cap_l);
    int l[D]; memset(l, 0, sizeof l);
    // simple recursive enumeration via stack
    int stackt = 0;
    // iterative: odometer over l_1..l_{D-1} with l_0 = j - sum
    memset(l, 0, sizeof l);
    for (;;) {
      int s = 0; for (int t = 1; t < D; ++t) s += l[t];
      if (s <= j) { l[0] = j - s; memcpy(L[cntj++], l, sizeof l); }
      int t = 1;
      while (t < D) { l[t]++; int s2 = 0; for (int u = 1; u < D; ++u) s2 += l[u]; if (s2 <= j) break; l[t] = 0; ++t; }
      if (t == D) break;
    }
    (void)stackt;
    double gc = 0, gs = 0, gl = 0; int ns = 0;
    for (int si = 0; si < (cntj < nsub ? cntj : nsub); ++si) {
      int sidx = cntj <= nsub ? si : (int)(sm64(rs++) % cntj);
      int* lv = L[sidx];
      for (int w = 0; w < nwarps; ++w) {
        uint64_t w0 = (sm64(rs++) % (m / 32)) * 32;
        uint32_t idx[32];
        for (int ln = 0; ln < 32; ++ln) {
          uint32_t q = kv[w0 + ln].q, v = 0;
          for (int t = 0; t < D; ++t) v = (v << lv[t]) | (uint32_t)(K[q * D + t] >> (NM - 1 - lv[t]));
          idx[ln] = v;
        }
        int cost = 0;
        for (int h = 0; h < 2; ++h) {
          int cnt[16] = {0};
          for (int a = 16 * h; a < 16 * h + 16; ++a) {
            int dup = 0;
            for (int b = 16 * h; b < a; ++b) if (idx[b] == idx[a]) { dup = 1; break; }
            if (!dup) cnt[idx[a] & 15]++;
          }
          int mx = 0; for (int k = 0; k < 16; ++k) if (cnt[k] > mx) mx = cnt[k];
          cost += mx;
        }
        int ds = 0, dl = 0;
        for (int a = 0; a < 32; ++a) {
          int dup = 0, dupl = 0;
          for (int b = 0; b < a; ++b) { if ((idx[b] >> 2) == (idx[a] >> 2)) dup = 1; if ((idx[b] >> 4) == (idx[a] >> 4)) dupl = 1; }
          ds += !dup; dl += !dupl;
        }
        gc += cost; gs += ds; gl += dl; ns++;
      }
    }
    gc /= ns; gs /= ns; gl /= ns;
    printf("group %2d: subspaces %6d  cycles/gather %.2f  sectors %.2f  lines %.2f\n", j, cntj, gc, gs, gl);
    tot_cost += gc * cntj; tot_sect += gs * cntj; tot_lines += gl * cntj; tot_terms += cntj;
    free(L);
  }
  printf("ALL: cycles/gather %.3f  sectors %.2f  lines %.2f  (ideal 2)\n", tot_cost / tot_terms, tot_sect / tot_terms,
         tot_lines / tot_terms);
  return 0;
}
