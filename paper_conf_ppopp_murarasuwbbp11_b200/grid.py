"""User-facing wrapper: ``Grid(d, n)`` owning an ``sg_grid`` handle.

    g = Grid(10, 11)                  # d = 10, level n = 11: 127,574,017 points
    x = g.coords()                    # grid-point coordinates (layout order)
    v = f(x)                          # sample the function to compress
    g.hierarchize_(v)                 # compression, in place: values -> surpluses
    y = g.evaluate(v, queries)        # decompression at arbitrary points

Compression/decompression as in the paper's application (Fig. 1).
All work happens in libsg's CUDA kernels; this class only owns the handle.
"""
from __future__ import annotations

import numpy as np
import torch

from . import _sg


class Grid:
    def __init__(self, d: int, n: int):
        self._h, self.num_points = _sg.sg_create(d, n)
        lay = _sg.sg_get_layout(self._h)
        self.d, self.n = d, n
        self.num_subspaces = lay["num_subspaces"]
        self.group_offset = lay["group_offset"]
        self.group_count = lay["group_count"]

    def close(self):
        if getattr(self, "_h", None) is not None:
            _sg.sg_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def handle(self):
        return self._h

    # ---- index maps (a8)
    def gp2idx(self, l, i):
        if isinstance(l, torch.Tensor) and l.is_cuda:
            out = torch.empty(l.shape[0], dtype=torch.int64, device=l.device)
            _sg.sg_gp2idx_device(self._h, l.contiguous(), i.contiguous(), out)
            return out
        return _sg.sg_gp2idx(self._h, np.asarray(l), np.asarray(i))

    def idx2gp(self, idx):
        if isinstance(idx, torch.Tensor) and idx.is_cuda:
            l = torch.empty((idx.numel(), self.d), dtype=torch.int32, device=idx.device)
            i = torch.empty_like(l)
            _sg.sg_idx2gp_device(self._h, idx.contiguous(), l, i)
            return l, i
        return _sg.sg_idx2gp(self._h, np.asarray(idx), self.d)

    def coords(self, first: int = 0, count: int | None = None, dtype=torch.float64, device="cuda"):
        count = self.num_points - first if count is None else count
        x = torch.empty((count, self.d), dtype=dtype, device=device)
        _sg.sg_grid_coords_device(self._h, first, count, x)
        return x

    # ---- compression (a7)
    def hierarchize_(self, values: torch.Tensor) -> torch.Tensor:
        if values.numel() != self.num_points:
            raise ValueError(f"values has {values.numel()} entries, the grid {self.num_points} points")
        _sg.sg_hierarchize(self._h, values)
        return values

    # ---- decompression (a1-a6)
    def workspace_bytes(self, m: int, dtype=torch.float64, presorted: bool = False) -> int:
        return _sg.sg_evaluate_workspace_bytes(self._h, m, dtype, _sg.SG_EVAL_PRESORTED if presorted else 0)

    def evaluate(self, alpha: torch.Tensor, x: torch.Tensor, out: torch.Tensor | None = None,
                 presorted: bool = False, workspace: torch.Tensor | None = None) -> torch.Tensor:
        _sg._check_batch(alpha, x, out, self.num_points, self.d)
        y = out if out is not None else torch.empty(x.shape[0], dtype=x.dtype, device=x.device)
        _sg.sg_evaluate(self._h, alpha, x.contiguous(), y, _sg.SG_EVAL_PRESORTED if presorted else 0, workspace)
        return y

    # ---- the multi-GPU building blocks: one global order, contiguous ranges of it
    def sfc_order(self, x: torch.Tensor, workspace: torch.Tensor | None = None) -> torch.Tensor:
        """Morton order of the batch (int32 permutation on x's device), identical on every rank."""
        _sg._check_batch(x, x, None, None, self.d)
        perm = torch.empty(x.shape[0], dtype=torch.int32, device=x.device)
        _sg.sg_sfc_order(self._h, x.contiguous(), perm, workspace)
        return perm

    def evaluate_ordered(self, alpha: torch.Tensor, x: torch.Tensor, perm: torch.Tensor | None, first: int,
                         count: int, out: torch.Tensor | None = None) -> torch.Tensor:
        """Evaluate positions first..first+count-1 of the order `perm`; out is the whole-batch result vector
        (input order) of which only those queries' entries are written."""
        _sg._check_batch(alpha, x, out, self.num_points, self.d)
        y = out if out is not None else torch.zeros(x.shape[0], dtype=x.dtype, device=x.device)
        _sg.sg_evaluate_ordered(self._h, alpha, x.contiguous(), perm, first, count, y)
        return y

    # ---- sharded grids (NEXT-4)
    def part_bounds(self, parts: int, part: int) -> tuple[int, int]:
        """(first, count): part `part` of `parts` contiguous, work-balanced ranges of the layout."""
        return _sg.sg_part_bounds(self._h, parts, part)

    def evaluate_part(self, alpha_part: torch.Tensor, parts: int, part: int, x: torch.Tensor,
                      out: torch.Tensor | None = None, perm: torch.Tensor | None = None,
                      accumulate: bool = False) -> torch.Tensor:
        """The part's share of f_s at every query (alpha_part = the part's surpluses only)."""
        first, count = self.part_bounds(parts, part)
        if alpha_part.numel() != count:
            raise ValueError(f"part {part}/{parts} holds {count} surpluses, got {alpha_part.numel()}")
        y = out if out is not None else torch.empty(x.shape[0], dtype=x.dtype, device=x.device)
        _sg.sg_evaluate_part(self._h, alpha_part, parts, part, x.contiguous(), y, perm, accumulate)
        return y

    # ---- visualization slice (NEXT-3)
    def render_plane(self, alpha: torch.Tensor, origin, du, dv, width: int, height: int, order: int = 1,
                     out: torch.Tensor | None = None, workspace: torch.Tensor | None = None) -> torch.Tensor:
        """(height, width) image of f_s at origin + (a+1/2) du + (b+1/2) dv (sg_evaluate_plane)."""
        if alpha.numel() != self.num_points:
            raise ValueError(f"alpha has {alpha.numel()} entries, the grid {self.num_points} points")
        for v in (origin, du, dv):
            if len(v) != self.d:
                raise ValueError(f"origin, du, dv need {self.d} entries")
        img = out if out is not None else torch.empty((height, width), dtype=alpha.dtype, device=alpha.device)
        _sg.sg_evaluate_plane(self._h, alpha, origin, du, dv, img, order, workspace)
        return img

    def evaluate_host(self, alpha: torch.Tensor, x_host, y_host=None, presorted: bool = False):
        if y_host is None:
            y_host = torch.empty(x_host.shape[0], dtype=x_host.dtype, pin_memory=True)
        _sg.sg_evaluate_host(self._h, alpha, x_host, y_host, _sg.SG_EVAL_PRESORTED if presorted else 0)
        return y_host


class BoundaryGrid:
    """Sparse grid with non-zero boundary (NEXT-2; paper Sec. 4.4, Fig. 7): the 3^d faces, each a
    zero-boundary sparse grid of its free dimensions (include/sg.h "NON-ZERO boundary")."""

    def __init__(self, d: int, n: int):
        self._h, self.num_points = _sg.sg_bcreate(d, n)
        self.d, self.n = d, n
        self.num_faces = 3 ** d

    def close(self):
        if getattr(self, "_h", None) is not None:
            _sg.sg_bdestroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def face(self, f: int) -> dict:
        mask, bits, first, count = _sg.sg_bface(self._h, f)
        return dict(free=[t for t in range(self.d) if mask >> t & 1], fixed_bits=bits, first=first, count=count)

    def coords(self, dtype=torch.float64, device="cuda") -> torch.Tensor:
        x = torch.empty((self.num_points, self.d), dtype=dtype, device=device)
        _sg.sg_bcoords_device(self._h, x)
        return x

    def hierarchize_(self, values: torch.Tensor) -> torch.Tensor:
        if values.numel() != self.num_points:
            raise ValueError(f"values has {values.numel()} entries, the grid {self.num_points} points")
        _sg.sg_bhierarchize(self._h, values)
        return values

    def evaluate(self, alpha: torch.Tensor, x: torch.Tensor, out: torch.Tensor | None = None) -> torch.Tensor:
        _sg._check_batch(alpha, x, out, self.num_points, self.d)
        y = out if out is not None else torch.empty(x.shape[0], dtype=x.dtype, device=x.device)
        _sg.sg_bevaluate(self._h, alpha, x.contiguous(), y)
        return y
