"""Pins for the CPU oracle (oracle/), independent of the oracle's own code.

Each test checks the oracle against something the paper or mathematics fixes,
never against a retyped copy of the oracle's formula:

  P1  point counts printed by the paper (golden/point_counts.txt, Fig. 3)
  P2  gp2idx/idx2gp: bijection onto [0, N) and equality with an independent,
      structural construction of the Sec. 4.1 layout
  P3  Alg. 3 order, first/last (eq. 3) and Alg. 4 next() = successor
  P4  Fig. 6 worked example (golden/fig6.txt)
  P5  closed-form surpluses of prod 4x(1-x) (golden/cfg1_surplus.txt) and of the
      cubic test function A (exact second difference)
  P6  interpolation invariant at grid points
  P7  combination technique (textbook identity; P:L749 names it)
  P8  separable DP for product functions (layout-free)
  P9  span reproduction: random surpluses -> values -> surpluses
  P10 d = 1: numpy.interp of the nodal values on the mesh 2^-n
  P11 d = 2: dense full-grid hierarchization restricted to the sparse grid
  O6  brute force over all N basis functions
"""
import itertools
import math

import numpy as np
import pytest

import sginputs as S
from conftest import all_points_structural, hat_np, read_golden

pytestmark = pytest.mark.filterwarnings("ignore")

SMALL_GRIDS = [(1, 1), (1, 6), (2, 1), (2, 3), (2, 5), (3, 4), (3, 5), (4, 4), (5, 4), (7, 3), (4, 6)]


# ---------------------------------------------------------------- P1 counts
def test_point_counts_printed_by_paper(oracle):
    for d, n, N, _cite in read_golden("point_counts.txt"):
        assert oracle.num_points(int(d), int(n)) == int(N)


@pytest.mark.parametrize("d,n", [(1, 5), (2, 4), (3, 5), (5, 4), (6, 3)])
def test_point_counts_brute_force(oracle, d, n):
    # sum over all level vectors with |l|_1 <= n-1 of 2^{|l|_1} (W_l has 2^|l| points)
    tot = sum(2 ** sum(l) for l in itertools.product(range(n), repeat=d) if sum(l) <= n - 1)
    assert oracle.num_points(d, n) == tot
    for j in range(n + 1):
        below = sum(2 ** sum(l) for l in itertools.product(range(n + 1), repeat=d) if sum(l) < j)
        assert oracle.index3(d, j) == below
    assert oracle.group_count(d, 3) == sum(1 for l in itertools.product(range(4), repeat=d) if sum(l) == 3)


def test_binomials_exact(oracle):
    for a in range(0, 66):
        for b in range(0, a + 1):
            assert oracle.binom(a, b) == math.comb(a, b)


# ---------------------------------------------------------------- P2 layout
@pytest.mark.parametrize("d,n", SMALL_GRIDS)
def test_layout_matches_structural_definition(oracle, d, n):
    L, I = all_points_structural(d, n)
    N = oracle.num_points(d, n)
    assert L.shape[0] == N
    idx = oracle.gp2idx(L, I)
    np.testing.assert_array_equal(idx, np.arange(N, dtype=np.uint64))
    l2, i2 = oracle.idx2gp(d, n, np.arange(N, dtype=np.uint64))
    np.testing.assert_array_equal(l2, L)
    np.testing.assert_array_equal(i2, I)


@pytest.mark.parametrize("d,n", [(3, 9), (6, 6), (10, 5), (20, 3)])
def test_roundtrip_bijection_bitmap(oracle, d, n):
    N = oracle.num_points(d, n)
    idx = np.arange(N, dtype=np.uint64)
    l, i = oracle.idx2gp(d, n, idx)
    assert np.all(l.sum(1) <= n - 1) and np.all(i % 2 == 1)
    assert np.all((i >= 1) & (i <= (1 << (l + 1)) - 1))
    back = oracle.gp2idx(l, i)
    np.testing.assert_array_equal(back, idx)
    # distinct (l, i) pairs: image is exactly [0, N)
    key = np.concatenate([l, i], axis=1)
    assert np.unique(key, axis=0).shape[0] == N
    with pytest.raises(IndexError):
        oracle.idx2gp(d, n, [N])


def test_roundtrip_cfg3_sample(oracle):
    d, n = 10, 11
    N = oracle.num_points(d, n)
    rng = np.random.default_rng(3)
    idx = np.unique(np.concatenate([rng.integers(0, N, 200000, dtype=np.uint64),
                                    np.arange(0, 5000, dtype=np.uint64),
                                    np.arange(N - 5000, N, dtype=np.uint64)]))
    l, i = oracle.idx2gp(d, n, idx)
    np.testing.assert_array_equal(oracle.gp2idx(l, i), idx)


# ---------------------------------------------------------------- P3 order
@pytest.mark.parametrize("d,j", [(2, 0), (2, 4), (3, 3), (4, 4), (5, 3), (6, 2)])
def test_alg3_order_first_last_next(oracle, d, j):
    E = oracle.enumerate_group(d, j)
    allv = [l for l in itertools.product(range(j + 1), repeat=d) if sum(l) == j]
    allv.sort(key=lambda l: tuple(reversed(l[1:])))
    np.testing.assert_array_equal(E, np.array(allv, dtype=np.int32).reshape(-1, d))
    # eq. (3): first(d, n) = (n, 0, ..., 0), last(d, n) = (0, ..., 0, n)
    first = np.zeros(d, np.int32); first[0] = j
    last = np.zeros(d, np.int32); last[-1] = j
    np.testing.assert_array_equal(E[0], first)
    np.testing.assert_array_equal(E[-1], last)
    # next(l) is the successor in this order (b - a = 1)
    for k in range(len(E) - 1):
        np.testing.assert_array_equal(oracle.next_level(E[k]), E[k + 1])
    assert oracle.next_level(E[-1]) is None


# ---------------------------------------------------------------- P4 Fig. 6
def test_fig6_worked_example(oracle):
    (l0, l1, i0, i1, x0, x1, printed, index3, index2, index1_fig, index1_alg5, pos) = read_golden("fig6.txt")[0]
    l = np.array([[int(l0), int(l1)]]); i = np.array([[int(i0), int(i1)]])
    got = int(oracle.gp2idx(l, i)[0])
    assert got == int(pos)
    assert got - int(index1_alg5) == int(index3) + int(index2) == int(printed) - int(index1_fig)
    assert oracle.index3(2, 3) == int(index3)
    # coordinates printed in the figure: x_t = i_t / 2^{l_t + 1}
    assert (int(i0) / 2 ** (int(l0) + 1), int(i1) / 2 ** (int(l1) + 1)) == (float(x0), float(x1))
    # Fig. 4: 1-based l=(1,2,2), i=(1,1,3) <-> (0.5, 0.25, 0.75); 0-based l=(0,1,1)
    lb, ib = np.array([0, 1, 1]), np.array([1, 1, 3])
    assert tuple(ib / 2.0 ** (lb + 1)) == (0.5, 0.25, 0.75)


# ---------------------------------------------------------------- P5 closed forms
def test_cfg1_closed_form_surpluses(oracle):
    d, n = 2, 3
    want = np.array([float(v) for row in read_golden("cfg1_surplus.txt") for v in row])
    x = oracle.coords(d, n)
    alpha = oracle.hierarchize(d, n, S.f_C(x))
    np.testing.assert_array_equal(alpha, want)


@pytest.mark.parametrize("d,n", [(1, 8), (2, 6), (3, 5), (5, 4)])
def test_closed_form_surpluses_quadratic(oracle, d, n):
    x = oracle.coords(d, n)
    l, _ = oracle.idx2gp(d, n, np.arange(x.shape[0], dtype=np.uint64))
    alpha = oracle.hierarchize(d, n, S.f_C(x))
    np.testing.assert_allclose(alpha, 4.0 ** (-l.sum(1).astype(float)), rtol=1e-13, atol=0)


@pytest.mark.parametrize("d,n", [(1, 9), (2, 7), (3, 6), (4, 5), (6, 4)])
def test_closed_form_surpluses_cubic_A(oracle, d, n):
    # g(x) = 4x(1-x)(1+cx) is cubic -> 1D surplus = -(h^2/2) g''(x) = 4^-l (1 - c + 3 c x)
    x = oracle.coords(d, n)
    l, _ = oracle.idx2gp(d, n, np.arange(x.shape[0], dtype=np.uint64))
    c = S.coeffs_A(d)
    want = np.prod(4.0 ** (-l.astype(float)) * (1.0 - c + 3.0 * c * x), axis=1)
    alpha = oracle.hierarchize(d, n, S.f_A(x))
    v = S.f_A(x)
    # absolute tolerance: v - (vL+vR)/2 cancels ~4^|l| of the value's ulps (SURVEY P5')
    np.testing.assert_allclose(alpha, want, rtol=0, atol=64 * d * np.finfo(float).eps * np.abs(v).max())
    assert np.all(alpha > 0)


# ---------------------------------------------------------------- P6 interpolation
@pytest.mark.parametrize("d,n", [(1, 6), (2, 5), (3, 4), (5, 3)])
def test_interpolation_invariant(oracle, d, n):
    x = oracle.coords(d, n)
    v = S.f_A(x)
    alpha = oracle.hierarchize(d, n, v)
    y, _ = oracle.evaluate(d, n, alpha, x)
    np.testing.assert_allclose(y, v, rtol=1e-14, atol=1e-16)


# ---------------------------------------------------------------- P7 combination technique
def _full_grid_interp(f, lvec, X):
    """Multilinear interpolant of f on the anisotropic full grid with mesh 2^-(l_t+1)
    in dimension t and zero boundary (the combination technique's component grids)."""
    m, d = X.shape
    out = np.zeros(m)
    h = 2.0 ** -(np.asarray(lvec) + 1.0)
    a = np.floor(X / h)
    w = X / h - a
    for corner in itertools.product((0, 1), repeat=d):
        cr = np.array(corner)
        node = (a + cr) * h
        wt = np.prod(np.where(cr == 1, w, 1.0 - w), axis=1)
        out += wt * f(node)
    return out


@pytest.mark.parametrize("d,n", [(2, 5), (3, 4), (4, 3)])
def test_combination_technique(oracle, d, n):
    X = S.queries(d, 300, seed=77 + d)
    alpha = oracle.hierarchize(d, n, S.f_A(oracle.coords(d, n)))
    y, _ = oracle.evaluate(d, n, alpha, X)
    ct = np.zeros(X.shape[0])
    for q in range(d):
        lev = n - 1 - q
        if lev < 0:
            continue
        for lvec in itertools.product(range(lev + 1), repeat=d):
            if sum(lvec) == lev:
                ct += (-1) ** q * math.comb(d - 1, q) * _full_grid_interp(S.f_A, lvec, X)
    np.testing.assert_allclose(y, ct, rtol=1e-13, atol=1e-15)


# ---------------------------------------------------------------- P8 separable DP
def separable_dp(d, n, X):
    """f_s(x) for f = prod g_t (function A): surpluses factor, so
    f_s = sum_{m<n} [z^m] prod_t (sum_l a_t(l) z^l), a_t(l) = s_t(l) phi_{l}(x_t)."""
    c = S.coeffs_A(d)
    m = X.shape[0]
    poly = np.zeros((m, n)); poly[:, 0] = 1.0
    for t in range(d):
        a = np.zeros((m, n))
        for lev in range(n):
            k = np.clip(np.floor(np.ldexp(X[:, t], lev)), 0, 2 ** lev - 1)
            centre = (2 * k + 1) / 2.0 ** (lev + 1)
            s = 4.0 ** -lev * (1.0 - c[t] + 3.0 * c[t] * centre)
            a[:, lev] = s * hat_np(lev, 2 * k + 1, X[:, t])
        new = np.zeros((m, n))
        for p in range(n):
            for q in range(n - p):
                new[:, p + q] += poly[:, p] * a[:, q]
        poly = new
    return poly.sum(1)


@pytest.mark.parametrize("d,n", [(2, 6), (4, 5), (6, 4), (10, 3)])
def test_separable_dp(oracle, d, n):
    X = S.queries(d, 500, seed=5 + d)
    alpha = oracle.hierarchize(d, n, S.f_A(oracle.coords(d, n)))
    y, ay = oracle.evaluate(d, n, alpha, X)
    np.testing.assert_allclose(y, separable_dp(d, n, X), rtol=1e-13, atol=0)
    np.testing.assert_allclose(ay, y, rtol=1e-15)  # positive surpluses: A(x) = |f_s(x)|


# ---------------------------------------------------------------- P9 span reproduction
@pytest.mark.parametrize("d,n", [(2, 5), (3, 4), (4, 3)])
def test_span_reproduction(oracle, d, n):
    N = oracle.num_points(d, n)
    alpha = S.random_surplus(N, seed=123)
    v, _ = oracle.evaluate(d, n, alpha, oracle.coords(d, n))
    back = oracle.hierarchize(d, n, v)
    np.testing.assert_allclose(back, alpha, rtol=0, atol=1e-13)


def test_single_basis_function(oracle):
    # one unit surplus reproduces exactly one hat function
    d, n = 3, 4
    N = oracle.num_points(d, n)
    X = S.queries(d, 200, seed=9)
    for j in [0, 5, N - 1]:
        alpha = np.zeros(N); alpha[j] = 1.0
        l, i = oracle.idx2gp(d, n, [j])
        want = np.prod([hat_np(l[0, t], i[0, t], X[:, t]) for t in range(d)], axis=0)
        y, _ = oracle.evaluate(d, n, alpha, X)
        np.testing.assert_allclose(y, want, rtol=4e-16, atol=0)


# ---------------------------------------------------------------- P10 d = 1
@pytest.mark.parametrize("n", [1, 4, 11])
def test_d1_piecewise_linear(oracle, n):
    xs = oracle.coords(1, n)[:, 0]
    v = np.sin(3.0 * xs) * xs * (1 - xs)
    alpha = oracle.hierarchize(1, n, v)
    X = S.queries(1, 1000, seed=1)
    y, _ = oracle.evaluate(1, n, alpha, X)
    order = np.argsort(xs)
    grid = np.concatenate([[0.0], xs[order], [1.0]])
    vals = np.concatenate([[0.0], v[order], [0.0]])
    np.testing.assert_allclose(y, np.interp(X[:, 0], grid, vals), rtol=0, atol=4e-16)


# ---------------------------------------------------------------- P11 d = 2 full grid
def _hier1d_dense(u, n, axis):
    u = np.moveaxis(u.copy(), axis, 0)
    for lev in range(n - 1, 0, -1):  # finest to coarsest, parents still nodal
        h = 2 ** (n - 1 - lev)
        pts = np.arange(h - 1, 2 ** n - 1, 2 * h)  # positions p with p+1 = odd * h
        left = np.where(pts - h >= 0, pts - h, -1)
        right = np.where(pts + h <= 2 ** n - 2, pts + h, -1)
        lv = np.where((left >= 0)[:, None], u[np.maximum(left, 0)], 0.0)
        rv = np.where((right >= 0)[:, None], u[np.maximum(right, 0)], 0.0)
        u[pts] = u[pts] - (lv + rv) / 2
    return np.moveaxis(u, 0, axis)


@pytest.mark.parametrize("n", [3, 5, 7])
def test_d2_dense_full_grid(oracle, n):
    g = (np.arange(1, 2 ** n) / 2.0 ** n)
    X0, X1 = np.meshgrid(g, g, indexing="ij")
    dense = S.f_A(np.stack([X0, X1], axis=-1))
    dense = _hier1d_dense(_hier1d_dense(dense, n, 0), n, 1)
    xs = oracle.coords(2, n)
    alpha = oracle.hierarchize(2, n, S.f_A(xs))
    pos = np.rint(xs * 2 ** n).astype(int) - 1
    np.testing.assert_array_equal(alpha, dense[pos[:, 0], pos[:, 1]])


# ---------------------------------------------------------------- O6 brute force, domain
@pytest.mark.parametrize("d,n", [(1, 5), (2, 4), (3, 3), (4, 3)])
def test_brute_force_equals_subspace_sum(oracle, d, n):
    N = oracle.num_points(d, n)
    alpha = S.random_surplus(N, seed=31)
    X = S.queries(d, 64, seed=32)
    y, ay = oracle.evaluate(d, n, alpha, X)
    np.testing.assert_allclose(oracle.evaluate_brute(d, n, alpha, X), y, rtol=0, atol=1e-15 * ay.max())


def test_outside_domain_and_nan(oracle):
    d, n = 3, 4
    N = oracle.num_points(d, n)
    alpha = S.random_surplus(N, seed=1)
    X = np.array([[0.0, 0.5, 0.5], [1.0, 0.5, 0.5], [-0.3, 0.2, 0.2], [0.5, 1.7, 0.5], [np.nan, 0.5, 0.5]])
    y, _ = oracle.evaluate(d, n, alpha, X)
    np.testing.assert_array_equal(y[:4], 0.0)
    assert np.isnan(y[4])
