"""CPU oracle for the compact sparse grid (Murarasu et al., PPoPP'11).

TEST INFRASTRUCTURE ONLY: only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA product path; see ``sg_oracle.c``
for the paper passage each function follows and DESIGN.md for the pins.

Every function takes/returns numpy arrays; levels are 0-based, the
grid parameter ``n`` is the number of level groups (paper "level n").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sg_oracle.c")
_LIB = os.path.join(_HERE, "libsg_oracle.so")


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2 -ffp-contract=off -fopenmp)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared", "-std=c11",
               "-Wall", "-Wextra", "-o", _LIB, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i32, p = ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p
        sig = {
            "or_binom": (u64, [i32, i32]),
            "or_group_count": (u64, [i32, i32]),
            "or_index3": (u64, [i32, i32]),
            "or_num_points": (u64, [i32, i32]),
            "or_enumerate": (u64, [i32, i32, p, u64]),
            "or_next": (i32, [i32, p, p]),
            "or_gp2idx": (u64, [i32, p, p]),
            "or_idx2gp": (i32, [i32, i32, u64, p, p]),
            "or_hierarchize": (None, [i32, i32, p]),
            "or_evaluate": (i32, [i32, i32, p, p, u64, p, p]),
            "or_evaluate_brute": (None, [i32, i32, p, p, u64, p]),
            "or_coords": (i32, [i32, i32, u64, u64, p]),
            "or_gp2idx_batch": (None, [i32, p, p, u64, p]),
            "or_idx2gp_batch": (i32, [i32, i32, p, u64, p, p]),
            "or_max_threads": (i32, []),
            "or_set_threads": (None, [i32]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def binom(a: int, b: int) -> int:
    return int(lib().or_binom(a, b))


def group_count(d: int, j: int) -> int:
    return int(lib().or_group_count(d, j))


def index3(d: int, j: int) -> int:
    return int(lib().or_index3(d, j))


def num_points(d: int, n: int) -> int:
    return int(lib().or_num_points(d, n))


def enumerate_group(d: int, j: int) -> np.ndarray:
    """Alg 3 order of L^d_j as an (S, d) int32 array."""
    cnt = group_count(d, j)
    out = np.zeros((cnt, d), dtype=np.int32)
    got = lib().or_enumerate(d, j, _ptr(out), cnt)
    assert got == cnt
    return out


def next_level(l) -> np.ndarray | None:
    """Alg 4 next(l); None for last(d, n) / the zero vector."""
    l = np.ascontiguousarray(l, dtype=np.int32)
    r = np.zeros_like(l)
    return None if lib().or_next(len(l), _ptr(l), _ptr(r)) else r


def gp2idx(l: np.ndarray, i: np.ndarray) -> np.ndarray:
    l = np.ascontiguousarray(np.atleast_2d(l), dtype=np.int32)
    i = np.ascontiguousarray(np.atleast_2d(i), dtype=np.int32)
    out = np.zeros(l.shape[0], dtype=np.uint64)
    lib().or_gp2idx_batch(l.shape[1], _ptr(l), _ptr(i), l.shape[0], _ptr(out))
    return out


def idx2gp(d: int, n: int, idx) -> tuple[np.ndarray, np.ndarray]:
    idx = np.ascontiguousarray(np.atleast_1d(idx), dtype=np.uint64)
    l = np.zeros((idx.size, d), dtype=np.int32)
    i = np.zeros((idx.size, d), dtype=np.int32)
    if lib().or_idx2gp_batch(d, n, _ptr(idx), idx.size, _ptr(l), _ptr(i)):
        raise IndexError("index out of range")
    return l, i


def coords(d: int, n: int, first: int = 0, count: int | None = None) -> np.ndarray:
    """Coordinates of grid points first..first+count-1 in layout order, (count, d)."""
    if count is None:
        count = num_points(d, n) - first
    x = np.zeros((count, d), dtype=np.float64)
    if lib().or_coords(d, n, first, count, _ptr(x)):
        raise IndexError("index out of range")
    return x


def hierarchize(d: int, n: int, values: np.ndarray) -> np.ndarray:
    """Alg 1 per pole per dimension; returns a new fp64 array of surpluses."""
    v = np.array(values, dtype=np.float64, copy=True)
    assert v.size == num_points(d, n)
    lib().or_hierarchize(d, n, _ptr(v))
    return v


def evaluate(d: int, n: int, alpha: np.ndarray, x: np.ndarray) -> tuple[np.ndarray, np.ndarray]:
    """(f_s(x_q), A(x_q) = sum |alpha phi|) for every row of x (widened to fp64)."""
    a = np.ascontiguousarray(alpha, dtype=np.float64)
    xx = np.ascontiguousarray(np.atleast_2d(x), dtype=np.float64)
    assert xx.shape[1] == d and a.size == num_points(d, n)
    y = np.zeros(xx.shape[0], dtype=np.float64)
    ay = np.zeros(xx.shape[0], dtype=np.float64)
    if lib().or_evaluate(d, n, _ptr(a), _ptr(xx), xx.shape[0], _ptr(y), _ptr(ay)):
        raise MemoryError("oracle evaluate: allocation failed")
    return y, ay


def evaluate_brute(d: int, n: int, alpha: np.ndarray, x: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(alpha, dtype=np.float64)
    xx = np.ascontiguousarray(np.atleast_2d(x), dtype=np.float64)
    y = np.zeros(xx.shape[0], dtype=np.float64)
    lib().or_evaluate_brute(d, n, _ptr(a), _ptr(xx), xx.shape[0], _ptr(y))
    return y


def max_threads() -> int:
    return int(lib().or_max_threads())


def set_threads(k: int) -> None:
    lib().or_set_threads(int(k))
