"""Pins of the non-zero-boundary oracle (oracle/boundary.py, Sec. 4.4 P:L461-L463,
Fig. 7) against what the paper and the mathematics fix, independently of its own code:

* the face counts the paper prints (2^j C(d, d-j) (d-j)-dimensional grids; Fig. 7: a 3d grid has 6 2d, 12 1d
  projections and 8 corners) and the resulting point count;
* multilinear functions prod_t (a_t + b_t x_t) lie in the span of the boundary basis (the corner functions
  prod (1-x) / x span them), so f_s = f EVERYWHERE, not only at the grid points;
* interpolation at every grid point (every face);
* d = 1: the piecewise-linear interpolant on the mesh 2^-n including the boundary values (numpy.interp);
* functions vanishing on the boundary: every boundary surplus is 0 and the interior surpluses are the
  (pinned) zero-boundary oracle's, bit for bit.
"""
import math

import numpy as np
import pytest

import sginputs as S


@pytest.fixture(scope="module")
def B(oracle):
    from oracle import boundary
    return boundary


@pytest.mark.parametrize("d", [1, 2, 3, 4, 5])
def test_face_counts_printed_by_paper(B, d):
    fs = B.faces(d)
    for k in range(d + 1):  # (d-k)-dimensional grids in the boundary: 2^k C(d, d-k)
        got = sum(1 for S_, _ in fs if len(S_) == d - k)
        want = 1 if k == 0 else 2 ** k * math.comb(d, d - k)
        assert got == want
    assert len(fs) == 3 ** d
    assert fs[0] == (tuple(range(d)), ())  # the interior first
    if d == 3:  # Fig. 7: 6 2d projections, 12 1d projections, 8 corners
        assert [sum(1 for S_, _ in fs if len(S_) == j) for j in (2, 1, 0)] == [6, 12, 8]


@pytest.mark.parametrize("d,n", [(1, 4), (2, 3), (3, 3), (2, 5)])
def test_point_count_closed_form(B, oracle, d, n):
    N = B.num_points(d, n)
    want = sum(math.comb(d, j) * 2 ** (d - j) * (1 if j == 0 else oracle.num_points(j, n)) for j in range(d + 1))
    assert N == want
    x, _, _, _ = B.points(d, n)
    assert x.shape == (N, d)
    assert len({tuple(r) for r in x.tolist()}) == N  # every point once


def multilinear(x, a, b):
    return np.prod(a[None, :] + b[None, :] * x, axis=1)


@pytest.mark.parametrize("d,n", [(1, 5), (2, 4), (3, 3), (4, 2)])
def test_multilinear_reproduced_everywhere(B, d, n):
    rng = np.random.default_rng(d * 10 + n)
    a, b = rng.random(d) + 0.5, rng.random(d) - 0.5
    xp, _, _, _ = B.points(d, n)
    alpha = B.hierarchize(d, n, multilinear(xp, a, b))
    xq = S.queries(d, 300, 5 + d)
    y, _ = B.evaluate(d, n, alpha, xq)
    np.testing.assert_allclose(y, multilinear(xq, a, b), rtol=1e-13, atol=1e-14)


@pytest.mark.parametrize("d,n", [(2, 4), (3, 3)])
def test_interpolation_at_every_point(B, d, n):
    xp, _, _, _ = B.points(d, n)
    f = np.sin(3.0 * xp.sum(1)) + xp[:, 0] ** 2
    alpha = B.hierarchize(d, n, f)
    y, _ = B.evaluate(d, n, alpha, xp)
    np.testing.assert_allclose(y, f, rtol=0, atol=1e-13)


@pytest.mark.parametrize("n", [1, 3, 6])
def test_d1_piecewise_linear_with_boundary_values(B, n):
    xp, _, _, _ = B.points(1, n)
    f = lambda t: np.cos(4.0 * t) + 0.5 * t
    alpha = B.hierarchize(1, n, f(xp[:, 0]))
    q = np.concatenate([S.queries(1, 500, 3)[:, 0], [0.0, 1.0]])
    y, _ = B.evaluate(1, n, alpha, q[:, None])
    knots = np.sort(xp[:, 0])
    np.testing.assert_allclose(y, np.interp(q, knots, f(knots)), rtol=0, atol=1e-14)


@pytest.mark.parametrize("d,n", [(2, 4), (3, 3)])
def test_zero_boundary_functions_match_the_zero_boundary_oracle(B, oracle, d, n):
    xp, fid, _, _ = B.points(d, n)
    vals = S.f_A(xp)  # vanishes on the boundary
    alpha = B.hierarchize(d, n, vals)
    Ni = oracle.num_points(d, n)
    assert np.all(fid[:Ni] == 0) and np.all(alpha[Ni:] == 0.0)
    np.testing.assert_array_equal(alpha[:Ni], oracle.hierarchize(d, n, vals[:Ni]))
