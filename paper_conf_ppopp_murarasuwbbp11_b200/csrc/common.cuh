// common.cuh -- shared internals of libsg (handle, errors, launch accounting).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <nvtx3/nvToolsExt.h>

#include <atomic>
#include <mutex>

#include "layout.cuh"

struct sg_grid_s {
  sg::Layout L;         // host tables
  int device;           // device that was current at sg_create
  sg::Layout* d_L;      // device copy of L
  // pole-family tables of the hierarchization (built on first use, per device
  // copy of the grid; hier_kernels.cu): per dimension, per family a packed
  // (|l_{-t}|, suffix sum) word and the offset of its first block base, and
  // per family per block the global offset of the block.  Built once, under
  // hier_mu and completed (stream-synchronised) before the pointer is
  // published, so concurrent callers on any stream see finished tables.
  mutable std::atomic<void*> d_hier_tab{nullptr};
  mutable std::mutex hier_mu;
};

namespace sg {

extern std::atomic<uint64_t> g_launches;
inline void count_launch(uint64_t k = 1) { g_launches.fetch_add(k, std::memory_order_relaxed); }

void set_error(const char* fmt, ...);
sg_status cuda_fail(cudaError_t e, const char* what);

// check the launch just issued; returns SG_OK or SG_ERR_CUDA
inline sg_status launched(const char* what) {
  count_launch();
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? SG_OK : cuda_fail(e, what);
}
// the same, recording WHICH kernel was launched (sg_launched_kernels: test instrumentation that checks every
// kernel in the library is exercised by the parity tests)
void record_kernel(const void* func);
inline sg_status launched(const char* what, const void* func) {
  record_kernel(func);
  return launched(what);
}

constexpr int kNumSMs = 148;

// NVTX range around one ABI call (header-only NVTX3: a no-op unless a profiler is attached), so that
// nsys/ncu timelines show the path's steps (a1 ordering, a2-a6 evaluation, a7 hierarchization, NEXT rows)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

// Function attributes are per device: opt a kernel into `smem` bytes of dynamic
// shared memory (and an L1/shared carveout, percent; < 0 = leave it) once per
// device, tracked in the caller's per-kernel bitmask (devices 0..63).
template <typename K>
inline sg_status set_smem_attr(K kern, std::atomic<uint64_t>& done, size_t smem, int carveout, const char* what) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, what);
  const uint64_t bit = 1ull << (dev & 63);
  if (done.load(std::memory_order_acquire) & bit) return SG_OK;
  e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)(smem > 48 * 1024 ? smem : 48 * 1024));
  if (e == cudaSuccess && carveout >= 0)
    e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, carveout > 100 ? 100 : carveout);
  if (e != cudaSuccess) return cuda_fail(e, what);
  done.fetch_or(bit, std::memory_order_release);
  return SG_OK;
}

// ---- kernel timing instrumentation (sg_profile_enable / sg_profile_read) ----
enum ProfKind { kProfEval = 0, kProfHier = 1 };
struct ProfScope {  // records an event pair around the launches in its lifetime when profiling is on
  cudaEvent_t a = nullptr, b = nullptr;
  cudaStream_t s;
  int kind;
  ProfScope(int kind_, cudaStream_t s_);
  ~ProfScope();
};  // B200; queried at run time where it matters

// ---- launchers implemented in the .cu files ---------------------------------
sg_status launch_gp2idx(const sg_grid_s* g, const int32_t* l, const int32_t* i, uint64_t count, uint64_t* idx,
                        cudaStream_t s);
sg_status launch_idx2gp(const sg_grid_s* g, const uint64_t* idx, uint64_t count, int32_t* l, int32_t* i,
                        cudaStream_t s);
sg_status launch_coords(const sg_grid_s* g, uint64_t first, uint64_t count, void* x, sg_dtype dt, cudaStream_t s);
sg_status launch_hierarchize(const sg_grid_s* g, void* v, sg_dtype dt, cudaStream_t s);
size_t sfc_workspace_bytes(uint64_t m);
sg_status launch_sfc_order(const sg_grid_s* g, const void* x, uint64_t m, sg_dtype dt, void* ws, size_t ws_bytes,
                           uint32_t* perm_dst, const uint32_t** perm_out, cudaStream_t s);
sg_status launch_evaluate(const sg_grid_s* g, const void* alpha, const void* x, const uint32_t* perm, uint64_t m,
                          void* y, sg_dtype dt, uint32_t flags, cudaStream_t s);
size_t plane_workspace_bytes(int d, uint64_t m, size_t elem);
// a part of the subspaces for the generic kernel (sharded grids): groups j0..j1, l_{d-1} from v0 in group
// j0 to v1 in group j1, running base starting at b0; accumulate adds to y
struct GenPart {
  int j0 = 0, v0 = 0, j1 = 64, v1 = 64;
  uint32_t b0 = 0;
  int accumulate = 0;
};
sg_status launch_plane(const sg_grid_s* g, const void* alpha, const double* origin, const double* du, const double* dv,
                       uint32_t width, uint32_t height, void* img, sg_dtype dt, uint32_t order, void* ws,
                       cudaStream_t s);

}  // namespace sg
