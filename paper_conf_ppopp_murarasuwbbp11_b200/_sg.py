"""Thin ctypes binding of libsg (include/sg.h): argument marshalling only.

Every function has the name of the C entry point it calls.  Device buffers
are torch tensors (their ``data_ptr()`` is passed); host buffers are numpy
arrays or CPU tensors.  The current torch CUDA stream is passed as the
``stream`` argument.  A non-SG_OK status raises :class:`SgError` carrying
``sg_last_error()``.  There is no fallback: if ``libsg.so`` is missing the
import fails.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np
import torch  # loads the CUDA runtime libsg links against

_HERE = os.path.dirname(os.path.abspath(__file__))
# SG_LIB selects another build of the same sources (scripts/gpu_exp.sh: libsg_exp.so); default: the product
LIB_PATH = os.environ.get("SG_LIB") or os.path.join(_HERE, "libsg.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built: run `python paper_conf_ppopp_murarasuwbbp11_b200/build.py` "
                      "(or __graft_entry__.build())")

lib = ctypes.CDLL(LIB_PATH)

SG_OK, SG_ERR_ARG, SG_ERR_RANGE, SG_ERR_OVERFLOW, SG_ERR_NOMEM, SG_ERR_CUDA, SG_ERR_DTYPE, SG_ERR_NODEV = range(8)
SG_F64, SG_F32 = 0, 1
SG_EVAL_PRESORTED = 1
SG_EVAL_GENERIC = 2
SG_MAX_D, SG_MAX_N = 32, 31

_u64, _i32, _u32, _p, _sz = ctypes.c_uint64, ctypes.c_int32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_size_t


class sg_layout(ctypes.Structure):
    _fields_ = [("d", ctypes.c_int32), ("n", ctypes.c_int32), ("num_points", ctypes.c_uint64),
                ("num_subspaces", ctypes.c_uint64), ("group_offset", ctypes.POINTER(ctypes.c_uint64)),
                ("group_count", ctypes.POINTER(ctypes.c_uint64))]


_SIGS = {
    "sg_create": [_i32, _i32, ctypes.POINTER(_p), ctypes.POINTER(_u64)],
    "sg_get_layout": [_p, ctypes.POINTER(sg_layout)],
    "sg_destroy": [_p],
    "sg_gp2idx": [_p, _p, _p, _u64, _p],
    "sg_idx2gp": [_p, _p, _u64, _p, _p],
    "sg_gp2idx_device": [_p, _p, _p, _u64, _p, _p],
    "sg_idx2gp_device": [_p, _p, _u64, _p, _p, _p],
    "sg_grid_coords_device": [_p, _u64, _u64, _p, ctypes.c_int, _p],
    "sg_hierarchize": [_p, _p, ctypes.c_int, _p],
    "sg_evaluate_workspace_bytes": [_p, _u64, ctypes.c_int, _u32, ctypes.POINTER(_sz)],
    "sg_evaluate": [_p, _p, _p, _u64, _p, ctypes.c_int, _u32, _p, _sz, _p],
    "sg_evaluate_host": [_p, _p, _p, _u64, _p, ctypes.c_int, _u32, _p],
    "sg_sfc_order": [_p, _p, _u64, ctypes.c_int, _p, _p, _sz, _p],
    "sg_evaluate_ordered": [_p, _p, _p, _u64, _p, _u64, _u64, _p, ctypes.c_int, _p],
    "sg_plane_workspace_bytes": [_p, _u32, _u32, ctypes.c_int, ctypes.POINTER(_sz)],
    "sg_part_bounds": [_p, _u32, _u32, ctypes.POINTER(_u64), ctypes.POINTER(_u64)],
    "sg_bcreate": [_i32, _i32, ctypes.POINTER(_p), ctypes.POINTER(_u64)],
    "sg_bdestroy": [_p],
    "sg_bface": [_p, _u32, ctypes.POINTER(_u32), ctypes.POINTER(_u32), ctypes.POINTER(_u64), ctypes.POINTER(_u64)],
    "sg_bcoords_device": [_p, _p, ctypes.c_int, _p],
    "sg_bhierarchize": [_p, _p, ctypes.c_int, _p],
    "sg_bevaluate": [_p, _p, _p, _u64, _p, ctypes.c_int, _p],
    "sg_evaluate_part": [_p, _p, _u32, _u32, _p, _u64, _p, _p, ctypes.c_int, ctypes.c_int, _p],
    "sg_evaluate_plane": [_p, _p, _p, _p, _p, _u32, _u32, _p, ctypes.c_int, _u32, _p, _sz, _p],
}
for _name, _args in _SIGS.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = ctypes.c_int
lib.sg_profile_enable.argtypes = [ctypes.c_int]
lib.sg_profile_enable.restype = ctypes.c_int
lib.sg_profile_read.argtypes = [ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_u64), ctypes.POINTER(ctypes.c_double),
                                ctypes.POINTER(_u64), ctypes.c_int]
lib.sg_profile_read.restype = ctypes.c_int
lib.sg_kernel_launch_count.restype = _u64
lib.sg_kernel_launch_count.argtypes = []
lib.sg_launched_kernels.restype = _sz
lib.sg_launched_kernels.argtypes = [ctypes.c_char_p, _sz]
for _name in ("sg_last_error", "sg_build_info"):
    getattr(lib, _name).restype = ctypes.c_char_p
    getattr(lib, _name).argtypes = []
lib.sg_status_string.restype = ctypes.c_char_p
lib.sg_status_string.argtypes = [ctypes.c_int]

#: every entry point declared in include/sg.h
EXPORTS = tuple(_SIGS) + ("sg_kernel_launch_count", "sg_status_string", "sg_last_error", "sg_build_info",
                          "sg_profile_enable", "sg_profile_read", "sg_launched_kernels")


class SgError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {lib.sg_status_string(status).decode()}: {lib.sg_last_error().decode()}")


def _check(status: int, where: str):
    if status != SG_OK:
        raise SgError(status, where)


def _dtype_code(t) -> int:
    dt = t.dtype if hasattr(t, "dtype") else t
    if dt in (torch.float64, np.float64):
        return SG_F64
    if dt in (torch.float32, np.float32):
        return SG_F32
    raise TypeError(f"unsupported dtype {dt}: libsg computes in float64 or float32")


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dev(t: torch.Tensor, name: str) -> int:
    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.is_contiguous()):
        raise ValueError(f"{name} must be a contiguous CUDA tensor")
    return t.data_ptr()


def _np_ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


# ------------------------------------------------------------------ calls
def sg_create(d: int, n: int):
    h = ctypes.c_void_p()
    N = ctypes.c_uint64()
    _check(lib.sg_create(d, n, ctypes.byref(h), ctypes.byref(N)), "sg_create")
    return h, int(N.value)


def sg_get_layout(g) -> dict:
    L = sg_layout()
    _check(lib.sg_get_layout(g, ctypes.byref(L)), "sg_get_layout")
    return dict(d=L.d, n=L.n, num_points=int(L.num_points), num_subspaces=int(L.num_subspaces),
                group_offset=[int(L.group_offset[k]) for k in range(L.n + 1)],
                group_count=[int(L.group_count[k]) for k in range(L.n)])


def sg_destroy(g) -> None:
    _check(lib.sg_destroy(g), "sg_destroy")


def sg_gp2idx(g, l: np.ndarray, i: np.ndarray) -> np.ndarray:
    """host gp2idx; raises SgError(SG_ERR_RANGE) if any item is not a grid point."""
    l = np.ascontiguousarray(np.atleast_2d(l), dtype=np.int32)
    i = np.ascontiguousarray(np.atleast_2d(i), dtype=np.int32)
    out = np.empty(l.shape[0], dtype=np.uint64)
    _check(lib.sg_gp2idx(g, _np_ptr(l), _np_ptr(i), l.shape[0], _np_ptr(out)), "sg_gp2idx")
    return out


def sg_idx2gp(g, idx: np.ndarray, d: int):
    idx = np.ascontiguousarray(np.atleast_1d(idx), dtype=np.uint64)
    l = np.empty((idx.size, d), dtype=np.int32)
    i = np.empty((idx.size, d), dtype=np.int32)
    _check(lib.sg_idx2gp(g, _np_ptr(idx), idx.size, _np_ptr(l), _np_ptr(i)), "sg_idx2gp")
    return l, i


def sg_gp2idx_device(g, l: torch.Tensor, i: torch.Tensor, idx: torch.Tensor, stream=None) -> None:
    assert l.dtype == torch.int32 and i.dtype == torch.int32 and idx.dtype in (torch.int64, torch.uint64)
    _check(lib.sg_gp2idx_device(g, _dev(l, "l"), _dev(i, "i"), l.shape[0], _dev(idx, "idx"), _stream(stream)),
           "sg_gp2idx_device")


def sg_idx2gp_device(g, idx: torch.Tensor, l: torch.Tensor, i: torch.Tensor, stream=None) -> None:
    assert l.dtype == torch.int32 and i.dtype == torch.int32 and idx.dtype in (torch.int64, torch.uint64)
    _check(lib.sg_idx2gp_device(g, _dev(idx, "idx"), idx.numel(), _dev(l, "l"), _dev(i, "i"), _stream(stream)),
           "sg_idx2gp_device")


def sg_grid_coords_device(g, first: int, count: int, x: torch.Tensor, stream=None) -> None:
    _check(lib.sg_grid_coords_device(g, first, count, _dev(x, "x"), _dtype_code(x), _stream(stream)),
           "sg_grid_coords_device")


def sg_hierarchize(g, values: torch.Tensor, stream=None) -> None:
    _check(lib.sg_hierarchize(g, _dev(values, "values"), _dtype_code(values), _stream(stream)), "sg_hierarchize")


def sg_evaluate_workspace_bytes(g, m: int, dtype, flags: int = 0) -> int:
    b = ctypes.c_size_t()
    _check(lib.sg_evaluate_workspace_bytes(g, m, _dtype_code(dtype), flags, ctypes.byref(b)),
           "sg_evaluate_workspace_bytes")
    return int(b.value)


def _check_batch(alpha: torch.Tensor, x: torch.Tensor, y: torch.Tensor | None = None, num_points: int | None = None,
                 d: int | None = None):
    """Shapes / dtypes / devices of one evaluation call (the C ABI takes raw pointers)."""
    if x.dim() != 2 or (d is not None and x.shape[1] != d):
        raise ValueError(f"x must be (m, {d if d is not None else 'd'}), got {tuple(x.shape)}")
    if alpha.dtype != x.dtype:
        raise ValueError(f"alpha ({alpha.dtype}) and x ({x.dtype}) must have the same dtype")
    if num_points is not None and alpha.numel() != num_points:
        raise ValueError(f"alpha has {alpha.numel()} entries, the grid {num_points} points")
    if y is not None:
        if y.dtype != x.dtype or y.numel() != x.shape[0] or not y.is_contiguous():
            raise ValueError(f"out must be a contiguous {x.dtype} tensor of {x.shape[0]} entries")
        if y.is_cuda != x.is_cuda or (y.is_cuda and y.device != x.device):
            raise ValueError("out must be on the same device as x")


def sg_evaluate(g, alpha: torch.Tensor, x: torch.Tensor, y: torch.Tensor, flags: int = 0,
                workspace: torch.Tensor | None = None, stream=None) -> None:
    _check_batch(alpha, x, y)
    ws = _dev(workspace, "workspace") if workspace is not None else None
    wsb = workspace.numel() * workspace.element_size() if workspace is not None else 0
    _check(lib.sg_evaluate(g, _dev(alpha, "alpha"), _dev(x, "x"), x.shape[0], _dev(y, "y"), _dtype_code(x), flags,
                           ws, wsb, _stream(stream)), "sg_evaluate")


def sg_sfc_order(g, x: torch.Tensor, perm: torch.Tensor, workspace: torch.Tensor | None = None, stream=None) -> None:
    """perm (m int32/uint32, device) <- the Morton order of the batch x (deterministic)."""
    if perm.dtype not in (torch.int32, torch.uint32) or perm.numel() != x.shape[0]:
        raise ValueError("perm must hold m int32 entries")
    ws = _dev(workspace, "workspace") if workspace is not None else None
    wsb = workspace.numel() * workspace.element_size() if workspace is not None else 0
    _check(lib.sg_sfc_order(g, _dev(x, "x"), x.shape[0], _dtype_code(x), _dev(perm, "perm"), ws, wsb,
                            _stream(stream)), "sg_sfc_order")


def sg_evaluate_ordered(g, alpha: torch.Tensor, x: torch.Tensor, perm: torch.Tensor | None, first: int, count: int,
                        y: torch.Tensor, stream=None) -> None:
    """y[perm[first+k]] = f_s(x[perm[first+k]]) for k < count (whole-batch x and y, input order)."""
    _check_batch(alpha, x, y)
    if perm is not None and (perm.dtype not in (torch.int32, torch.uint32) or perm.numel() != x.shape[0]):
        raise ValueError("perm must hold m int32 entries")
    pp = _dev(perm, "perm") if perm is not None else None
    _check(lib.sg_evaluate_ordered(g, _dev(alpha, "alpha"), _dev(x, "x"), x.shape[0], pp, first, count, _dev(y, "y"),
                                   _dtype_code(x), _stream(stream)), "sg_evaluate_ordered")


def sg_plane_workspace_bytes(g, width: int, height: int, dtype) -> int:
    b = ctypes.c_size_t()
    _check(lib.sg_plane_workspace_bytes(g, width, height, _dtype_code(dtype), ctypes.byref(b)),
           "sg_plane_workspace_bytes")
    return int(b.value)


def sg_evaluate_plane(g, alpha: torch.Tensor, origin, du, dv, image: torch.Tensor, order: int = 1,
                      workspace: torch.Tensor | None = None, stream=None) -> None:
    """image (height, width) <- f_s on the plane origin + (a+1/2) du + (b+1/2) dv."""
    if image.dim() != 2 or image.dtype != alpha.dtype:
        raise ValueError("image must be a (height, width) tensor of alpha's dtype")
    h, w = image.shape
    o = np.ascontiguousarray(origin, dtype=np.float64)
    u = np.ascontiguousarray(du, dtype=np.float64)
    v = np.ascontiguousarray(dv, dtype=np.float64)
    ws = _dev(workspace, "workspace") if workspace is not None else None
    wsb = workspace.numel() * workspace.element_size() if workspace is not None else 0
    _check(lib.sg_evaluate_plane(g, _dev(alpha, "alpha"), _np_ptr(o), _np_ptr(u), _np_ptr(v), w, h,
                                 _dev(image, "image"), _dtype_code(alpha), order, ws, wsb, _stream(stream)),
           "sg_evaluate_plane")


def sg_part_bounds(g, parts: int, part: int) -> tuple[int, int]:
    first, count = ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib.sg_part_bounds(g, parts, part, ctypes.byref(first), ctypes.byref(count)), "sg_part_bounds")
    return int(first.value), int(count.value)


def sg_evaluate_part(g, alpha_part: torch.Tensor, parts: int, part: int, x: torch.Tensor, y: torch.Tensor,
                     perm: torch.Tensor | None = None, accumulate: bool = False, stream=None) -> None:
    _check_batch(alpha_part, x, y)
    pp = _dev(perm, "perm") if perm is not None else None
    ap = _dev(alpha_part, "alpha_part") if alpha_part.numel() else None
    _check(lib.sg_evaluate_part(g, ap, parts, part, _dev(x, "x"), x.shape[0], pp, _dev(y, "y"), 1 if accumulate else 0,
                                _dtype_code(x), _stream(stream)), "sg_evaluate_part")


def sg_bcreate(d: int, n: int):
    h = ctypes.c_void_p()
    N = ctypes.c_uint64()
    _check(lib.sg_bcreate(d, n, ctypes.byref(h), ctypes.byref(N)), "sg_bcreate")
    return h, int(N.value)


def sg_bdestroy(g) -> None:
    _check(lib.sg_bdestroy(g), "sg_bdestroy")


def sg_bface(g, face: int) -> tuple[int, int, int, int]:
    m, b, f, c = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib.sg_bface(g, face, ctypes.byref(m), ctypes.byref(b), ctypes.byref(f), ctypes.byref(c)), "sg_bface")
    return int(m.value), int(b.value), int(f.value), int(c.value)


def sg_bcoords_device(g, x: torch.Tensor, stream=None) -> None:
    _check(lib.sg_bcoords_device(g, _dev(x, "x"), _dtype_code(x), _stream(stream)), "sg_bcoords_device")


def sg_bhierarchize(g, values: torch.Tensor, stream=None) -> None:
    _check(lib.sg_bhierarchize(g, _dev(values, "values"), _dtype_code(values), _stream(stream)), "sg_bhierarchize")


def sg_bevaluate(g, alpha: torch.Tensor, x: torch.Tensor, y: torch.Tensor, stream=None) -> None:
    _check_batch(alpha, x, y)
    _check(lib.sg_bevaluate(g, _dev(alpha, "alpha"), _dev(x, "x"), x.shape[0], _dev(y, "y"), _dtype_code(x),
                            _stream(stream)), "sg_bevaluate")


def sg_evaluate_host(g, alpha: torch.Tensor, x_host, y_host, flags: int = 0, stream=None) -> None:
    """x_host / y_host: CPU tensors (pinned for full copy bandwidth) or numpy arrays."""
    if x_host.shape[0] != y_host.shape[0] or x_host.dtype != y_host.dtype or x_host.dtype != alpha.dtype:
        raise ValueError("x_host (m, d) and y_host (m) must match alpha's dtype and each other's length")
    xp = x_host.data_ptr() if isinstance(x_host, torch.Tensor) else x_host.ctypes.data
    yp = y_host.data_ptr() if isinstance(y_host, torch.Tensor) else y_host.ctypes.data
    _check(lib.sg_evaluate_host(g, _dev(alpha, "alpha"), xp, x_host.shape[0], yp, _dtype_code(x_host), flags,
                                _stream(stream)), "sg_evaluate_host")


def sg_kernel_launch_count() -> int:
    return int(lib.sg_kernel_launch_count())


def sg_launched_kernels() -> list[str]:
    """Mangled names of the distinct libsg kernels launched since load (test instrumentation)."""
    need = int(lib.sg_launched_kernels(None, 0))
    buf = ctypes.create_string_buffer(need)
    lib.sg_launched_kernels(buf, need)
    return [s for s in buf.value.decode().split("\n") if s]


def sg_build_info() -> str:
    return lib.sg_build_info().decode()


def sg_profile_enable(on: bool) -> None:
    _check(lib.sg_profile_enable(1 if on else 0), "sg_profile_enable")


def sg_profile_read(reset: bool = False) -> dict:
    em, hm = ctypes.c_double(), ctypes.c_double()
    en, hn = ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib.sg_profile_read(ctypes.byref(em), ctypes.byref(en), ctypes.byref(hm), ctypes.byref(hn),
                               1 if reset else 0), "sg_profile_read")
    return dict(eval_ms=em.value, eval_launches=int(en.value), hier_ms=hm.value, hier_launches=int(hn.value))
