"""Seeded synthetic workloads shared by the oracle side and the CUDA side.

This module holds ONLY input generation: a counter-based random generator
(SplitMix64), query batches, random surplus vectors and the analytic test
functions that are sampled at grid points.  It contains none of the sparse-grid
method's arithmetic (no level/index maps, no hat functions, no layout), so both
`oracle/` and the CUDA path may import it without sharing method code
(see DESIGN.md "Inputs").

Recipes:

* queries: ``x[q, t] = ((splitmix64(seed ^ (q*d + t)) >> 11) + 0.5) * 2**-53``,
  every coordinate in the open interval (0, 1) and a multiple of 2**-54; the
  paper evaluates at 10^5 points "in the domain" without stating a
  distribution (reading G16: uniform).
* cfg4 plane: ``x0 = (a + 0.5)/W``, ``x1 = (b + 0.5)/H``, ``x2 = 0.3``
  (reading G19), row-major with ``a`` fastest.
* random surpluses (source B): ``alpha_j = 2 * U(splitmix64(seed ^ j)) - 1``.
* test function A: ``prod_t 4 x_t (1 - x_t) (1 + c_t x_t)``,
  ``c_t = (t + 1) / (2 d + 2)``; test function C: ``prod_t 4 x_t (1 - x_t)``.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)

#: BASELINE.json configs (cfg2p is SURVEY G18's n=10 variant of cfg2).
CONFIGS = {
    "cfg1": dict(d=2, n=3, m=1000, dtype="f64", source="C", seed=0x5EED0001),
    "cfg2": dict(d=5, n=8, m=1_000_000, dtype="f64", source="A", seed=0x5EED0002),
    "cfg2p": dict(d=5, n=10, m=1_000_000, dtype="f64", source="A", seed=0x5EED0012),
    "cfg3": dict(d=10, n=11, m=10_000_000, dtype="f64", source="A", seed=0x5EED0003),
    "cfg4": dict(d=3, n=14, m=4096 * 4096, dtype="f32", source="A", seed=0x5EED0004,
                 plane=(4096, 4096, 0.3)),
    "cfg5": dict(d=20, n=6, m=1_000_000, dtype="f64", source="A", seed=0x5EED0005),
}


def splitmix64(v: np.ndarray) -> np.ndarray:
    """SplitMix64 output function applied to counters ``v`` (uint64, wraps)."""
    z = np.asarray(v, dtype=np.uint64) + GOLDEN
    z = (z ^ (z >> np.uint64(30))) * M1
    z = (z ^ (z >> np.uint64(27))) * M2
    return z ^ (z >> np.uint64(31))


def _unit_open(bits: np.ndarray) -> np.ndarray:
    """Map uint64 to a double in (0, 1): ((b >> 11) + 0.5) * 2^-53 (exact)."""
    return ((bits >> np.uint64(11)).astype(np.float64) + 0.5) * (2.0 ** -53)


def queries(d: int, m: int, seed: int, first: int = 0, dtype=np.float64,
            chunk: int = 1 << 22) -> np.ndarray:
    """Row-major ``(m, d)`` query batch, rows ``first .. first+m-1`` of the stream."""
    out = np.empty((m, d), dtype=dtype)
    s = np.uint64(seed)
    t = np.arange(d, dtype=np.uint64)
    for q0 in range(0, m, chunk):
        q1 = min(m, q0 + chunk)
        q = np.arange(first + q0, first + q1, dtype=np.uint64)[:, None]
        ctr = (q * np.uint64(d) + t[None, :]) ^ s
        out[q0:q1] = _unit_open(splitmix64(ctr)).astype(dtype)
    return out


def plane_queries(width: int, height: int, x2: float, d: int = 3, dtype=np.float32) -> np.ndarray:
    """cfg4 visualisation slice: pixel centres of a width x height plane at x_2 = x2."""
    a = (np.arange(width, dtype=np.float64) + 0.5) / width
    b = (np.arange(height, dtype=np.float64) + 0.5) / height
    out = np.empty((height, width, d), dtype=np.float64)
    out[:, :, 0] = a[None, :]
    out[:, :, 1] = b[:, None]
    for t in range(2, d):
        out[:, :, t] = x2
    return out.reshape(width * height, d).astype(dtype)


def random_surplus(num: int, seed: int, first: int = 0, dtype=np.float64) -> np.ndarray:
    """Source B: alpha_j = 2 U_j - 1 with U_j from splitmix64(seed ^ j)."""
    j = np.arange(first, first + num, dtype=np.uint64)
    return (2.0 * _unit_open(splitmix64(j ^ np.uint64(seed))) - 1.0).astype(dtype)


def coeffs_A(d: int) -> np.ndarray:
    return (np.arange(d, dtype=np.float64) + 1.0) / (2.0 * d + 2.0)


def f_A(x: np.ndarray) -> np.ndarray:
    """Separable non-symmetric test function A (zero on the boundary).

    Written as one elementwise op at a time, dimension by dimension, so that
    the numpy and torch versions round identically."""
    x = np.asarray(x, dtype=np.float64)
    d = x.shape[-1]
    r = np.ones(x.shape[:-1], dtype=np.float64)
    for t in range(d):
        xt = x[..., t]
        c = (t + 1.0) / (2.0 * d + 2.0)
        g = ((4.0 * xt) * (1.0 - xt)) * (1.0 + c * xt)
        r = r * g
    return r


def f_C(x: np.ndarray) -> np.ndarray:
    """cfg1 test function prod_t 4 x_t (1 - x_t)."""
    x = np.asarray(x, dtype=np.float64)
    r = np.ones(x.shape[:-1], dtype=np.float64)
    for t in range(x.shape[-1]):
        xt = x[..., t]
        r = r * ((4.0 * xt) * (1.0 - xt))
    return r


# ---- torch variants (same streams, generated on any device) -----------------

def _t_splitmix64(v):
    def s64(c):  # unsigned constant -> int64 two's complement
        return c - (1 << 64) if c >= (1 << 63) else c

    def lsr(z, k):  # logical shift right on int64
        return (z >> k) & ((1 << (64 - k)) - 1)

    z = v + s64(0x9E3779B97F4A7C15)
    z = (z ^ lsr(z, 30)) * s64(0xBF58476D1CE4E5B9)
    z = (z ^ lsr(z, 27)) * s64(0x94D049BB133111EB)
    return z ^ lsr(z, 31)


def queries_torch(d: int, m: int, seed: int, device, dtype=None, first: int = 0,
                  chunk: int = 1 << 22):
    """Same stream as :func:`queries`, produced with torch ops on ``device``."""
    import torch
    dtype = dtype or torch.float64
    out = torch.empty((m, d), dtype=dtype, device=device)
    s = seed - (1 << 64) if seed >= (1 << 63) else seed
    t = torch.arange(d, dtype=torch.int64, device=device)
    for q0 in range(0, m, chunk):
        q1 = min(m, q0 + chunk)
        q = torch.arange(first + q0, first + q1, dtype=torch.int64, device=device)[:, None]
        z = _t_splitmix64((q * d + t[None, :]) ^ s)
        hi = (z >> 11) & ((1 << 53) - 1)
        out[q0:q1] = ((hi.to(torch.float64) + 0.5) * (2.0 ** -53)).to(dtype)
    return out


def random_surplus_torch(num: int, seed: int, device, dtype=None, chunk: int = 1 << 24):
    import torch
    dtype = dtype or torch.float64
    out = torch.empty(num, dtype=dtype, device=device)
    s = seed - (1 << 64) if seed >= (1 << 63) else seed
    for j0 in range(0, num, chunk):
        j1 = min(num, j0 + chunk)
        j = torch.arange(j0, j1, dtype=torch.int64, device=device)
        z = _t_splitmix64(j ^ s)
        hi = (z >> 11) & ((1 << 53) - 1)
        out[j0:j1] = (2.0 * ((hi.to(torch.float64) + 0.5) * (2.0 ** -53)) - 1.0).to(dtype)
    return out


def f_A_torch(x):
    import torch
    xd = x.to(torch.float64)
    d = xd.shape[-1]
    r = torch.ones(xd.shape[:-1], dtype=torch.float64, device=xd.device)
    for t in range(d):
        xt = xd[..., t]
        c = (t + 1.0) / (2.0 * d + 2.0)
        g = ((4.0 * xt) * (1.0 - xt)) * (1.0 + c * xt)
        r = r * g
    return r


def f_C_torch(x):
    import torch
    xd = x.to(torch.float64)
    r = torch.ones(xd.shape[:-1], dtype=torch.float64, device=xd.device)
    for t in range(xd.shape[-1]):
        xt = xd[..., t]
        r = r * ((4.0 * xt) * (1.0 - xt))
    return r
