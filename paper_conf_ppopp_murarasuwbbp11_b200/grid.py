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
        assert values.numel() == self.num_points
        _sg.sg_hierarchize(self._h, values)
        return values

    # ---- decompression (a1-a6)
    def workspace_bytes(self, m: int, dtype=torch.float64, presorted: bool = False) -> int:
        return _sg.sg_evaluate_workspace_bytes(self._h, m, dtype, _sg.SG_EVAL_PRESORTED if presorted else 0)

    def evaluate(self, alpha: torch.Tensor, x: torch.Tensor, out: torch.Tensor | None = None,
                 presorted: bool = False, workspace: torch.Tensor | None = None) -> torch.Tensor:
        assert x.dim() == 2 and x.shape[1] == self.d and x.dtype == alpha.dtype
        y = out if out is not None else torch.empty(x.shape[0], dtype=x.dtype, device=x.device)
        _sg.sg_evaluate(self._h, alpha, x.contiguous(), y, _sg.SG_EVAL_PRESORTED if presorted else 0, workspace)
        return y

    def evaluate_host(self, alpha: torch.Tensor, x_host, y_host=None, presorted: bool = False):
        if y_host is None:
            y_host = torch.empty(x_host.shape[0], dtype=x_host.dtype, pin_memory=True)
        _sg.sg_evaluate_host(self._h, alpha, x_host, y_host, _sg.SG_EVAL_PRESORTED if presorted else 0)
        return y_host
