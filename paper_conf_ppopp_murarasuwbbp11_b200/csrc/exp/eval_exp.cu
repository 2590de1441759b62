// eval_exp.cu -- EXPERIMENT variants of the evaluation kernel, compiled only into libsg_exp.so
// (build.py --exp; never into the product libsg.so).  Selected at run time by SG_EXP_VAR; used by
// scripts/gpu_exp.sh to measure what bounds the product kernel.
#include <stdlib.h>
#include <string.h>

#include "../eval_trie.cuh"

namespace sg {

struct KnobsGO : trie::Knobs {
  static constexpr bool GO = true;
};
struct KnobsLZ3 : trie::Knobs {
  static constexpr bool LZ3 = true;
};

// GO: gather-only (all hat values 1; same addresses, loads and Horner adds), cfg3 shape
template <int MINB, int NT = 128>
static sg_status d10_go(const Layout& L, const double* a, const double* x, const uint32_t* p, uint64_t m, double* y,
                        cudaStream_t s) {
  sg_status st = SG_OK;
#define SG_R(J0, J1) \
  if (st == SG_OK) st = trie::launch_range<double, 10, 11, NT, MINB, J0, J1, KnobsGO>(L, a, x, p, m, y, s);
  SG_R(0, 6) SG_R(7, 7) SG_R(8, 8) SG_R(9, 9) SG_R(10, 10)
#undef SG_R
  return st;
}

sg_status exp_SY9(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);
sg_status exp_LIDBL(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);
sg_status exp_SIDBL(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);
sg_status exp_GOT(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);

sg_status exp_SP20(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);
sg_status exp_D20ID(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);
sg_status exp_SP20B(const Layout&, const double*, const double*, const uint32_t*, uint64_t, double*, cudaStream_t);
// returns true if an experiment variant handled the call (the variants measured in r01/r02 before v9 are
// recorded in profiles/r02_split.txt and profiles/r02_cfg5_variants.txt; their code is in the git history)
bool exp_dispatch(const Layout& L, const void* alpha, const void* x, const uint32_t* perm, uint64_t m, void* y,
                  sg_dtype dt, cudaStream_t s, sg_status* st) {
  const char* v = getenv("SG_EXP_VAR");
  if (!v) return false;
  if (dt != SG_F64) return false;
  if (L.d == 20 && L.n <= 6) {
    const double* a = (const double*)alpha;
    if (!strcmp(v, "SP20")) { *st = exp_SP20(L, a, (const double*)x, perm, m, (double*)y, s); return true; }
    if (!strcmp(v, "D20ID")) { *st = exp_D20ID(L, a, (const double*)x, perm, m, (double*)y, s); return true; }
    if (!strcmp(v, "SP20B")) { *st = exp_SP20B(L, a, (const double*)x, perm, m, (double*)y, s); return true; }
    return false;
  }
  if (L.d != 10 || L.n != 11) return false;
  const double* a = (const double*)alpha;
  const double* xx = (const double*)x;
  double* yy = (double*)y;
  if (!strcmp(v, "GO4")) { *st = d10_go<4>(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SY9")) { *st = exp_SY9(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "LIDBL")) { *st = exp_LIDBL(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "SIDBL")) { *st = exp_SIDBL(L, a, xx, perm, m, yy, s); return true; }
  if (!strcmp(v, "GOT")) { *st = exp_GOT(L, a, xx, perm, m, yy, s); return true; }
  return false;
}

}  // namespace sg
