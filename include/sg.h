/*
 * sg.h -- C ABI of libsg, a B200 (sm_100a) implementation of the compact
 * sparse-grid data structure and its compression/decompression algorithms
 * from Murarasu, Weidendorfer, Buse, Butnaru, Pflueger: "Compact Data Structure
 * and Scalable Algorithms for the Sparse Grid Technique", PPoPP'11.
 * Citations "P:L<n>" refer to lines of the paper text.
 *
 * Problem statement: compression = computing the hierarchical
 * coefficients (surpluses) alpha_{l,i} from function values at the sparse-grid
 * points ("hierarchization"); decompression = evaluating
 *      f_s(x) = sum_{|l|_1 <= n-1} sum_i alpha_{l,i} phi_{l,i}(x)
 * anywhere in [0,1]^d ("evaluation").  Surpluses live in one flat array in
 * the paper's bijective layout gp2idx (Sec. 4.1-4.2).
 *
 * Conventions used by every call:
 *  - Levels are 0-based as in the paper from Sec. 4 on.  The grid
 *    parameter n is the paper's "level n" (level 11 <-> 127,574,017
 *    points at d = 10); the grid holds the level groups j = |l|_1 = 0..n-1.
 *  - A grid point is (l, i): l_t >= 0, i_t odd in [1, 2^{l_t+1}-1], at
 *    coordinate x_t = i_t / 2^{l_t+1}; phi_{l,i}(x) = prod_t
 *    max(0, 1 - |2^{l_t+1} x_t - i_t|), zero boundary.
 *  - Layout: idx = index3 + index2 + index1:
 *      index3 = number of points of all groups j' < |l|_1
 *      index2 = subspaceidx(l) * 2^{|l|_1}, subspaceidx = eq. (4),
 *               i.e. the rank of l in the Alg. 3 order
 *      index1 = position of i in subspace l, dimension 0 most significant
 *               (Alg. 5 line 3; reading G2 on Fig. 6).
 *  - Level vectors / indices are int32 arrays of `count x d`, row-major.
 *  - Query points are `m x d` row-major; values/surpluses/results are fp64
 *    (SG_F64) or fp32 (SG_F32); every buffer of one call has the same dtype.
 *  - "device" pointers are CUDA device pointers on the device that was current
 *    at sg_create; "host" pointers are host memory (pinned recommended).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    Device calls are stream-ordered and asynchronous unless stated otherwise.
 *  - Ownership: the caller owns every data buffer and workspace; the library
 *    owns the grid handle and its small per-device tables (freed by
 *    sg_destroy).  No call keeps a pointer to caller memory after it returns
 *    (asynchronous calls read/write it in stream order).
 *  - Errors: every call returns sg_status; nothing throws across the ABI.
 *    SG_ERR_CUDA carries the CUDA error text in sg_last_error() (thread-local).
 */
#ifndef SG_H
#define SG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SG_MAX_D 32 /* maximum dimension */
#define SG_MAX_N 31 /* maximum number of level groups (finest 1D level n-1 <= 30) */

/* sg_evaluate flags */
#define SG_EVAL_PRESORTED 1u /* skip the space-filling-curve ordering of the queries (a1) */
#define SG_EVAL_GENERIC 2u   /* force the generic (unspecialised) evaluation kernel; for testing */

typedef struct sg_grid_s *sg_grid; /* opaque; immutable after sg_create; may be shared by threads */

typedef enum {
  SG_OK = 0,
  SG_ERR_ARG = 1,      /* invalid argument (NULL pointer, bad d/n/dtype, short workspace) */
  SG_ERR_RANGE = 2,    /* some batch item is not a grid point / index >= N (sentinel written) */
  SG_ERR_OVERFLOW = 3, /* the grid has >= 2^62 points */
  SG_ERR_NOMEM = 4,    /* host or device allocation failed */
  SG_ERR_CUDA = 5,     /* a CUDA call failed; see sg_last_error() */
  SG_ERR_DTYPE = 6,    /* unsupported dtype */
  SG_ERR_NODEV = 7     /* no CUDA device / the library was not built for it */
} sg_status;

typedef enum { SG_F64 = 0, SG_F32 = 1 } sg_dtype;

typedef struct {
  int32_t d, n;
  uint64_t num_points;          /* N = sum_{j<n} 2^j C(d-1+j, d-1) */
  uint64_t num_subspaces;       /* sum_{j<n} C(d-1+j, d-1) = C(n-1+d, d)   (terms per evaluation) */
  const uint64_t *group_offset; /* n+1 host entries: index3(j), group_offset[n] = N        */
  const uint64_t *group_count;  /* n host entries: |L^d_j| = C(d-1+j, d-1)  (eq. 2) */
} sg_layout;

/* Create the grid of dimension d (1..SG_MAX_D) and level n (1..SG_MAX_N),
 * build its tables (binomial matrix "binmat" and index3 offsets) and
 * upload them to the current CUDA device.  *out receives the handle,
 * *num_points (may be NULL) the number of points N.  Without a CUDA device
 * the handle is host-only: sg_get_layout, sg_gp2idx and sg_idx2gp work and
 * every device call returns SG_ERR_NODEV. */
sg_status sg_create(int32_t d, int32_t n, sg_grid *out, uint64_t *num_points);

/* Layout description; the pointers stay valid until sg_destroy. */
sg_status sg_get_layout(sg_grid g, sg_layout *out);

/* Release the handle and its device tables (synchronizes the device). */
sg_status sg_destroy(sg_grid g);

/* gp2idx (Alg. 5) on HOST memory: idx[k] = gp2idx(l[k,:], i[k,:]).
 * Items that are not grid points of g get idx = UINT64_MAX and the call
 * returns SG_ERR_RANGE (the other items are still written). Synchronous. */
sg_status sg_gp2idx(sg_grid g, const int32_t *l, const int32_t *i, uint64_t count, uint64_t *idx);

/* idx2gp (inverse of gp2idx) on HOST memory.  Indices >= N get
 * l = i = -1 in all d entries and the call returns SG_ERR_RANGE. Synchronous. */
sg_status sg_idx2gp(sg_grid g, const uint64_t *idx, uint64_t count, int32_t *l, int32_t *i);

/* Device-batch versions of the two maps (same semantics, one CUDA kernel
 * each, asynchronous).  Invalid items get the same sentinels; because the
 * call is asynchronous the return value reports argument errors only -- use
 * the sentinels to detect range errors. */
sg_status sg_gp2idx_device(sg_grid g, const int32_t *d_l, const int32_t *d_i, uint64_t count,
                           uint64_t *d_idx, void *stream);
sg_status sg_idx2gp_device(sg_grid g, const uint64_t *d_idx, uint64_t count, int32_t *d_l, int32_t *d_i,
                           void *stream);

/* Coordinates of the grid points first..first+count-1 (layout order) into
 * d_x (count x d, dtype dt): x_t = i_t / 2^{l_t+1}, exact.  Used to sample the
 * function to compress ("select only the function values at grid points",
 * P:L253).  first+count must be <= N. */
sg_status sg_grid_coords_device(sg_grid g, uint64_t first, uint64_t count, void *d_x, sg_dtype dt,
                                void *stream);

/* Compression (hierarchization, Alg. 1 / Alg. 6):
 * d_values holds N nodal values f(x_j) in layout order on entry and the N
 * surpluses alpha_j on exit (in place).  Dimensions are processed t = 0..d-1
 * (reading G10); each point's update is  v - (v_left + v_right)/2  with the
 * left/right 1D hierarchical parents' values of the previous pass (0 on the
 * boundary).  Uses no workspace for n <= 14 (fp64) / n <= 15 (fp32); larger
 * grids allocate N values of scratch with cudaMallocAsync on `stream`. */
sg_status sg_hierarchize(sg_grid g, void *d_values, sg_dtype dt, void *stream);

/* Bytes of device workspace sg_evaluate needs for m queries (0 with
 * SG_EVAL_PRESORTED). */
sg_status sg_evaluate_workspace_bytes(sg_grid g, uint64_t m, sg_dtype dt, uint32_t flags, size_t *bytes);

/* Decompression (evaluation, Alg. 7):
 *   d_y[q] = f_s(d_x[q,:]) = sum_j d_alpha[j] phi_j(d_x[q,:]),  q < m.
 * d_alpha: N surpluses in layout order; d_x: m x d; d_y: m; all on the device
 * and of dtype dt.  Unless SG_EVAL_PRESORTED, the queries are first ordered
 * along a Morton curve (a device sort inside the call) and results are
 * scattered back, so d_y is always in input order.  d_workspace must hold
 * sg_evaluate_workspace_bytes bytes; pass NULL/0 to let the call allocate it
 * stream-ordered (cudaMallocAsync).  Any real x is accepted: f_s = 0 outside
 * (0,1)^d and on the boundary; a NaN coordinate gives NaN. */
sg_status sg_evaluate(sg_grid g, const void *d_alpha, const void *d_x, uint64_t m, void *d_y, sg_dtype dt,
                      uint32_t flags, void *d_workspace, size_t ws_bytes, void *stream);

/* Row a1 on its own: the space-filling-curve order of a query batch.
 * d_perm (m uint32, device, caller-owned) receives the permutation that
 * sorts d_x (m x d, dtype dt) along the Morton curve sg_evaluate uses (the
 * paper's blocking over evaluation points; coalesced coordinate
 * staging).  The sort is a stable radix sort of (key, index) pairs,
 * so the result is a deterministic function of the batch: every process that
 * orders the same batch obtains the same permutation (multi-GPU ranks agree
 * on one global order without communicating).  d_workspace must
 * hold sg_evaluate_workspace_bytes(g, m, dt, 0) bytes, or be NULL (allocated
 * stream-ordered).  Asynchronous on `stream`. */
sg_status sg_sfc_order(sg_grid g, const void *d_x, uint64_t m, sg_dtype dt, uint32_t *d_perm, void *d_workspace,
                       size_t ws_bytes, void *stream);

/* Evaluate one contiguous range of an ordered batch (the multi-GPU shard of
 * the "embarrassingly parallel" evaluation, Sec. 4.3, with a static
 * workload distribution):
 *   for k < count:  q = d_perm[first + k];  d_y[q] = f_s(d_x[q,:]).
 * d_x (m x d) and d_y (m) are the WHOLE batch in input order (only the
 * range's rows of d_x are read and only its entries of d_y written);
 * d_perm (m entries) is an order from sg_sfc_order.  With d_perm == NULL the
 * batch is taken as already ordered: rows first..first+count-1.  The result
 * of every query is bitwise independent of the range it is evaluated in.
 * first + count must be <= m (SG_ERR_RANGE otherwise).  Asynchronous. */
sg_status sg_evaluate_ordered(sg_grid g, const void *d_alpha, const void *d_x, uint64_t m, const uint32_t *d_perm,
                              uint64_t first, uint64_t count, void *d_y, sg_dtype dt, void *stream);

/* Visualization slice (the paper's motivating application, interactive visualization
 * of compressed data, Fig. 1; evaluation "at arbitrary locations"): renders
 * d_image[b * width + a] = f_s(x(a, b)),  x(a, b) = origin + (a + 1/2) du + (b + 1/2) dv,
 * for pixel columns a < width and rows b < height, each coordinate rounded as
 * fl(fl(origin_t + (a+1/2) du_t) + (b+1/2) dv_t) in fp64, then converted to dt.  origin, du, dv are HOST
 * arrays of d doubles (copied at the call).  order 0 visits the pixels in row-major order, order 1 in
 * 8 x 4 warp tiles along a 2D Morton curve of the tiles (needs width % 8 == 0 and height % 4 == 0, else
 * row-major).  No query array is needed: the pixel coordinates and the visiting order are generated on the
 * device into d_workspace (sg_plane_workspace_bytes bytes, or NULL: allocated stream-ordered).  The values
 * are bitwise those of sg_evaluate at the same points.  Asynchronous. */
sg_status sg_plane_workspace_bytes(sg_grid g, uint32_t width, uint32_t height, sg_dtype dt, size_t *bytes);
sg_status sg_evaluate_plane(sg_grid g, const void *d_alpha, const double *origin, const double *du, const double *dv,
                            uint32_t width, uint32_t height, void *d_image, sg_dtype dt, uint32_t order,
                            void *d_workspace, size_t ws_bytes, void *stream);

/* Grids sharded across devices (the paper's evaluation is a sum over subspaces,
 * Alg. 7, so it splits into partial sums over disjoint subspace sets).  The layout is cut
 * into `parts` contiguous index ranges at (level group j, level l_{d-1}) boundaries -- whole groups for
 * d <= 5 -- each holding about 1/parts of the subspaces, i.e. of the evaluation work.
 * sg_part_bounds: the range [*first, *first + *count) of part `part` (host only, any grid).
 * sg_evaluate_part: d_y[q] (+)= the part's share of f_s(x_q), q < m (accumulate != 0 adds to d_y),
 * with d_alpha_part holding ONLY the part's *count surpluses (alpha[first .. first+count)); summing the
 * parts' results (e.g. one NCCL all-reduce) gives f_s up to rounding.  d_perm (may be NULL) orders the
 * queries as in sg_evaluate_ordered.  Generic kernels only: d <= 12, n <= 12, N < 2^32 (SG_ERR_ARG
 * otherwise).  Asynchronous. */
sg_status sg_part_bounds(sg_grid g, uint32_t parts, uint32_t part, uint64_t *first, uint64_t *count);
sg_status sg_evaluate_part(sg_grid g, const void *d_alpha_part, uint32_t parts, uint32_t part, const void *d_x,
                           uint64_t m, const uint32_t *d_perm, void *d_y, int accumulate, sg_dtype dt, void *stream);

/* ---- Sparse grids with NON-ZERO boundary (Sec. 4.4, Fig. 7).
 * "The boundary of a d-dimensional sparse grid is composed of lower-dimensional, zero-boundary sparse grids":
 * the grid is the list of the 3^d FACES (S, c) -- S the free dimensions, c in {0,1}^{d-|S|} the values of
 * the fixed ones -- each carrying the |S|-dimensional zero-boundary grid of level n (the interior is S = all,
 * the corners |S| = 0: one point).  Layout (reading G20; the paper leaves the ordering function open):
 * faces grouped by dimensionality |S| = d, d-1, ..., 0, inside a group by the free-dimension bitmask
 * ascending, then by the fixed values as a binary number (bit k = value of the k-th fixed dimension);
 * inside a face the |S|-dimensional layout above over the free dimensions in increasing order.
 * Basis: phi_p(x) = prod_{t in S} phi_{l_t,i_t}(x_t) prod_{t not in S} b_{c_t}(x_t), b_0(x) = 1-x, b_1(x) = x
 * on [0,1]; f_s = 0 outside [0,1]^d; NaN propagates.  1 <= d <= 12, 1 <= n <= 14.
 * sg_bcreate/sg_bdestroy: the handle (host layout; device tables when a GPU is present).
 * sg_bface: the layout of face `face` (< 3^d): free mask, fixed bits, first index, point count.
 * sg_bcoords_device: the coordinates (N x d, layout order) of every point, exact.
 * sg_bhierarchize: in place, nodal values -> surpluses, dimension by dimension (t = 0..d-1): every point of
 *   a face with t free becomes v - (v_L + v_R)/2 with its 1D parents at x_t -+ 2^-(l_t+1) (on the face
 *   fixing t to 0 / 1 when the parent coordinate is 0 / 1), values of pass t-1.
 * sg_bevaluate: d_y[q] = sum_faces prod_{t fixed} b_{c_t}(x_t) f_face(x_S), each f_face through the
 *   zero-boundary evaluation path.  All device calls are asynchronous on `stream`. */
typedef struct sg_bgrid_s *sg_bgrid;
sg_status sg_bcreate(int32_t d, int32_t n, sg_bgrid *out, uint64_t *num_points);
sg_status sg_bdestroy(sg_bgrid g);
sg_status sg_bface(sg_bgrid g, uint32_t face, uint32_t *free_mask, uint32_t *fixed_bits, uint64_t *first,
                   uint64_t *count);
sg_status sg_bcoords_device(sg_bgrid g, void *d_x, sg_dtype dt, void *stream);
sg_status sg_bhierarchize(sg_bgrid g, void *d_values, sg_dtype dt, void *stream);
sg_status sg_bevaluate(sg_bgrid g, const void *d_alpha, const void *d_x, uint64_t m, void *d_y, sg_dtype dt,
                       void *stream);

/* End-to-end evaluation from HOST buffers: copies h_x (m x d) to the device,
 * evaluates as sg_evaluate, copies the m results to h_y.  d_alpha is on the
 * device.  Device buffers are allocated stream-ordered.  The three steps run
 * back to back on `stream` (H2D of the whole batch, evaluation, D2H): the
 * space-filling-curve order needs every query on the device before the
 * first evaluation launch, and chunking the batch would shrink the warps'
 * spatial locality.  Returns after the results are in
 * h_y (synchronizes `stream`). */
sg_status sg_evaluate_host(sg_grid g, const void *d_alpha, const void *h_x, uint64_t m, void *h_y, sg_dtype dt,
                           uint32_t flags, void *stream);

/* Number of CUDA kernels the library launched since load (instrumentation
 * for the bench's gpu_launches count). */
uint64_t sg_kernel_launch_count(void);

/* Test instrumentation: the (mangled) names of the distinct kernels the library launched since load,
 * newline-separated, into buf (at most len bytes incl. the terminating 0); returns the bytes needed. */
size_t sg_launched_kernels(char *buf, size_t len);

/* Kernel timing instrumentation.  While enabled (on != 0), every evaluation
 * kernel launch and every hierarchization pass is bracketed by CUDA events
 * recorded on the launching stream.  sg_profile_read synchronizes on those
 * events and returns the summed device milliseconds and launch counts since
 * the last reset (reset != 0 clears them).  Any pointer may be NULL. */
sg_status sg_profile_enable(int on);
sg_status sg_profile_read(double *eval_ms, uint64_t *eval_launches, double *hier_ms, uint64_t *hier_launches,
                          int reset);

const char *sg_status_string(sg_status s);
const char *sg_last_error(void); /* thread-local detail of the last error ("" if none) */
const char *sg_build_info(void); /* compile flags / target architecture */

#ifdef __cplusplus
}
#endif
#endif /* SG_H */
