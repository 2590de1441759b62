// eval_trie.cu -- dispatch of the v2 evaluation kernel (eval_trie.cuh) by
// (d, n, dtype); shapes without an instantiation return handled = false and
// fall through to eval_gen.cuh (generic run-time-level kernels) / eval_simple.cu.
#include "common.cuh"

namespace sg {

#define SG_DECL(name, T) \
  sg_status name(const Layout& L, const T* a, const T* x, const uint32_t* p, uint64_t m, T* y, cudaStream_t s);
SG_DECL(trie_d10n11_a, double)
SG_DECL(trie_d10n11_b, double)
SG_DECL(trie_d2n3, double)
SG_DECL(trie_d5n8, double)
SG_DECL(trie_d5n10, double)
SG_DECL(trie_d3n14f, float)
SG_DECL(trie_d20n6, double)
#undef SG_DECL
#ifdef SG_EXP
bool exp_dispatch(const Layout& L, const void* alpha, const void* x, const uint32_t* perm, uint64_t m, void* y,
                  sg_dtype dt, cudaStream_t s, sg_status* st);
#endif

sg_status launch_eval_trie(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                           void* y, sg_dtype dt, cudaStream_t s, bool* handled) {
  *handled = false;
  if (m > 0xffffffffull || g->L.N >= 0xffffffffull) return SG_OK;  // 32-bit offsets
  const Layout& L = g->L;
  const int d = L.d, n = L.n;
  *handled = true;
#ifdef SG_EXP
  {
    sg_status st = SG_OK;
    if (exp_dispatch(L, alpha, x, perm, m, y, dt, s, &st)) return st;
  }
#endif
  if (dt == SG_F64) {
    const double* a = (const double*)alpha;
    const double* xx = (const double*)x;
    double* yy = (double*)y;
    // each instantiation serves every n up to its level bound (launches of groups >= n are skipped)
    if (d == 10 && n <= 11) {
      sg_status st = trie_d10n11_a(L, a, xx, perm, m, yy, s);
      if (st != SG_OK) return st;
      return trie_d10n11_b(L, a, xx, perm, m, yy, s);
    }
    if (d == 2 && n <= 3) return trie_d2n3(L, a, xx, perm, m, yy, s);
    if (d == 5 && n <= 8) return trie_d5n8(L, a, xx, perm, m, yy, s);
    if (d == 5 && n <= 10) return trie_d5n10(L, a, xx, perm, m, yy, s);
    if (d == 20 && n <= 6) return trie_d20n6(L, a, xx, perm, m, yy, s);
  } else {
    if (d == 3 && n <= 14) return trie_d3n14f(L, (const float*)alpha, (const float*)x, perm, m, (float*)y, s);
  }
  *handled = false;
  return SG_OK;
}

}  // namespace sg
