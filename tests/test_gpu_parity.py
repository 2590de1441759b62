"""GPU parity: every CUDA kernel behind include/sg.h against the CPU oracle on
the same seeded inputs (BASELINE.json configs).

  index maps, coordinates, hierarchization (fp64): bit-exact
  evaluation: |y - y_oracle| <= tol * A(x), A(x) = sum |alpha phi| (normwise,
      reading G13), tol = 1e-12 (fp64) / 1e-5 (fp32); with positive surpluses
      (function A) A(x) = |f_s(x)| and this is plain relative error.
  full size (cfg3, 10^7 queries, the launch configuration bench.py times):
      the oracle on a seeded sample of queries, plus every output against the
      layout-free separable closed form (pin P8).
"""
import ctypes

import numpy as np
import pytest

import sginputs as S
from conftest import gpu_available

pytestmark = [pytest.mark.gpu, pytest.mark.skipif(not gpu_available(), reason="needs a CUDA device")]

TOL = {"f64": 1e-12, "f32": 1e-5}


@pytest.fixture(scope="module")
def P():
    import paper_conf_ppopp_murarasuwbbp11_b200 as P
    return P


@pytest.fixture(scope="module")
def torch():
    import torch
    return torch


def tdt(torch, dt):
    return torch.float64 if dt == "f64" else torch.float32


def check_eval(y_gpu, y_ref, a_ref, tol, what=""):
    y_gpu = np.asarray(y_gpu, dtype=np.float64)
    err = np.abs(y_gpu - y_ref)
    scale = np.maximum(a_ref, np.finfo(float).tiny)
    worst = np.max(err / scale) if err.size else 0.0
    assert worst <= tol, f"{what}: normwise error {worst:.3e} > {tol:.0e}"
    return worst


def hierarchized_alpha(torch, P, g, source, dt, seed=0):
    """Surpluses on the device: function A/C sampled at the grid points and
    hierarchized by sg_hierarchize, or random surpluses (source B)."""
    if source == "B":
        return S.random_surplus_torch(g.num_points, seed=seed, device="cuda", dtype=tdt(torch, dt))
    x = g.coords(dtype=torch.float64)
    v = (S.f_A_torch(x) if source == "A" else S.f_C_torch(x)).to(tdt(torch, dt))
    del x
    return g.hierarchize_(v)


# ----------------------------------------------------------------- index maps
@pytest.mark.parametrize("d,n", [(1, 8), (2, 5), (3, 6), (5, 5), (10, 4), (20, 3), (32, 2)])
def test_device_index_maps_all_points(P, torch, oracle, d, n):
    g = P.Grid(d, n)
    N = g.num_points
    idx = torch.arange(N, dtype=torch.int64, device="cuda")
    l, i = g.idx2gp(idx)
    lo, io = oracle.idx2gp(d, n, np.arange(N, dtype=np.uint64))
    np.testing.assert_array_equal(l.cpu().numpy(), lo)
    np.testing.assert_array_equal(i.cpu().numpy(), io)
    back = g.gp2idx(torch.from_numpy(lo).cuda(), torch.from_numpy(io).cuda())
    np.testing.assert_array_equal(back.cpu().numpy(), np.arange(N))
    x = g.coords()
    np.testing.assert_array_equal(x.cpu().numpy(), oracle.coords(d, n))


def test_device_index_maps_cfg3_every_point(P, torch, oracle):
    d, n = 10, 11
    g = P.Grid(d, n)
    N = g.num_points
    seen = torch.zeros(N, dtype=torch.int32, device="cuda")
    chunk = 1 << 24
    for a in range(0, N, chunk):
        idx = torch.arange(a, min(N, a + chunk), dtype=torch.int64, device="cuda")
        l, i = g.idx2gp(idx)
        back = g.gp2idx(l, i)
        assert torch.equal(back, idx)
        seen.index_add_(0, back, torch.ones_like(back, dtype=torch.int32))
    assert int(seen.min()) == 1 and int(seen.max()) == 1  # image is exactly [0, N)
    rng = np.random.default_rng(5)
    samp = rng.integers(0, N, 200000).astype(np.uint64)
    l, i = g.idx2gp(torch.from_numpy(samp.astype(np.int64)).cuda())
    lo, io = oracle.idx2gp(d, n, samp)
    np.testing.assert_array_equal(l.cpu().numpy(), lo)
    np.testing.assert_array_equal(i.cpu().numpy(), io)


def test_device_sentinels(P, torch):
    g = P.Grid(3, 4)
    idx = torch.tensor([0, g.num_points, -1], dtype=torch.int64, device="cuda")
    l, i = g.idx2gp(idx)
    assert (l[1:] == -1).all() and (i[1:] == -1).all() and (l[0] == 0).all()
    lv = torch.tensor([[0, 0, 0], [4, 0, 0], [0, 0, 1]], dtype=torch.int32, device="cuda")
    iv = torch.tensor([[1, 1, 1], [1, 1, 1], [1, 1, 4]], dtype=torch.int32, device="cuda")
    out = g.gp2idx(lv, iv)
    assert out[0].item() == 0 and out[1].item() == -1 and out[2].item() == -1


# ----------------------------------------------------------------- hierarchization
@pytest.mark.parametrize("d,n", [(1, 1), (1, 11), (2, 3), (2, 8), (3, 7), (5, 8), (6, 6), (10, 5), (20, 4),
                                 (3, 14)])
def test_hierarchize_bit_exact_fp64(P, torch, oracle, d, n):
    g = P.Grid(d, n)
    xs = oracle.coords(d, n)
    v = S.f_A(xs) + 0.25 * np.sin(7.0 * xs.sum(1))  # not separable, not symmetric
    want = oracle.hierarchize(d, n, v)
    got = g.hierarchize_(torch.from_numpy(v).cuda()).cpu().numpy()
    np.testing.assert_array_equal(got, want)


def test_hierarchize_table_reuse_and_fp32(P, torch, oracle):
    """The pole-family tables are built on the first call and reused: a second
    and third hierarchization on the same handle (other data, other dtype)
    stay bit-exact / within fp32 rounding of the oracle."""
    d, n = 4, 7
    g = P.Grid(d, n)
    xs = oracle.coords(d, n)
    for k in range(2):
        v = S.f_A(xs) * (1.0 + k) + 0.1 * np.cos((3.0 + k) * xs.sum(1))
        got = g.hierarchize_(torch.from_numpy(v).cuda()).cpu().numpy()
        np.testing.assert_array_equal(got, oracle.hierarchize(d, n, v))
    v32 = (S.f_A(xs) - 0.2 * np.sin(2.0 * xs.prod(1))).astype(np.float32)
    got32 = g.hierarchize_(torch.from_numpy(v32).cuda()).cpu().numpy().astype(np.float64)
    want = oracle.hierarchize(d, n, v32.astype(np.float64))
    np.testing.assert_allclose(got32, want, rtol=0, atol=64 * d * np.finfo(np.float32).eps * np.abs(v32).max())


@pytest.mark.parametrize("d,n,dt", [(1, 17, "f64"), (2, 15, "f64"), (1, 17, "f32")])
def test_hierarchize_large_families_fallback(P, torch, oracle, d, n, dt):
    # 2^n - 1 values per pole family exceed shared memory: global ping-pong kernel
    g = P.Grid(d, n)
    xs = oracle.coords(d, n)
    v = S.f_A(xs) + 0.25 * np.cos(5.0 * xs.sum(1))
    if dt == "f32":
        v32 = v.astype(np.float32)
        want = oracle.hierarchize(d, n, v32.astype(np.float64))
        got = g.hierarchize_(torch.from_numpy(v32).cuda()).cpu().numpy().astype(np.float64)
        np.testing.assert_allclose(got, want, rtol=0, atol=64 * d * np.finfo(np.float32).eps * np.abs(v32).max())
        return
    want = oracle.hierarchize(d, n, v)
    got = g.hierarchize_(torch.from_numpy(v).cuda()).cpu().numpy()
    np.testing.assert_array_equal(got, want)


def test_hierarchize_cfg1_golden(P, torch):
    from conftest import read_golden
    g = P.Grid(2, 3)
    alpha = hierarchized_alpha(torch, P, g, "C", "f64")
    want = np.array([float(v) for row in read_golden("cfg1_surplus.txt") for v in row])
    np.testing.assert_array_equal(alpha.cpu().numpy(), want)


def test_hierarchize_fp32_cfg4_grid(P, torch, oracle):
    d, n = 3, 14
    g = P.Grid(d, n)
    xs = oracle.coords(d, n)
    v32 = S.f_A(xs).astype(np.float32)
    want = oracle.hierarchize(d, n, v32.astype(np.float64))
    got = g.hierarchize_(torch.from_numpy(v32).cuda()).cpu().numpy().astype(np.float64)
    atol = 64 * d * np.finfo(np.float32).eps * np.abs(v32).max()
    np.testing.assert_allclose(got, want, rtol=0, atol=atol)


def test_hierarchize_cfg3_bit_exact_vs_oracle(P, torch, oracle):
    """The full cfg3 compression (127,574,017 points, the bench workload) bit-exact against the oracle's
    Alg. 1 pole recursion (reading G10: dimensions 0..d-1; x0.5 is exact, so FMA contraction cannot
    change a bit), on function A plus a non-separable term."""
    d, n = 10, 11
    g = P.Grid(d, n)
    vals = torch.empty(g.num_points, dtype=torch.float64, device="cuda")
    for a in range(0, g.num_points, 1 << 23):
        b = min(g.num_points, a + (1 << 23))
        xc = g.coords(a, b - a)
        vals[a:b] = S.f_A_torch(xc) + 0.25 * torch.sin(7.0 * xc.sum(1))
    host = vals.cpu().numpy()
    got = g.hierarchize_(vals).cpu().numpy()
    want = oracle.hierarchize(d, n, host)
    assert np.array_equal(got, want)


def test_hierarchize_cfg3_closed_form(P, torch, oracle):
    """Full cfg3 grid (127.6M points) against the closed-form surpluses of the
    cubic function A (pin P5'): every surplus positive, a 10^6 sample exact to
    an absolute bound, on the indices' (l, i) from the oracle."""
    d, n = 10, 11
    g = P.Grid(d, n)
    alpha = hierarchized_alpha(torch, P, g, "A", "f64")
    assert bool((alpha > 0).all())
    rng = np.random.default_rng(17)
    samp = np.unique(rng.integers(0, g.num_points, 1_000_000).astype(np.uint64))
    l, i = oracle.idx2gp(d, n, samp)
    x = i / 2.0 ** (l + 1)
    c = S.coeffs_A(d)
    want = np.prod(4.0 ** (-l.astype(float)) * (1.0 - c + 3.0 * c * x), axis=1)
    got = alpha[torch.from_numpy(samp.astype(np.int64)).cuda()].cpu().numpy()
    np.testing.assert_allclose(got, want, rtol=0, atol=64 * d * np.finfo(float).eps * 1.5)


# ----------------------------------------------------------------- evaluation
CASES = [
    # name, source, oracle sample size
    ("cfg1", "C", None),
    ("cfg2", "A", 4000),
    ("cfg2", "B", 2000),
    ("cfg2p", "A", 1000),
    ("cfg5", "A", 160),
    ("cfg5", "B", 100),
    ("cfg4", "A", 4000),
]


def config_queries(torch, cfg, dt):
    c = S.CONFIGS[cfg]
    if "plane" in c:
        w, h, x2 = c["plane"]
        xq = S.plane_queries(w, h, x2, d=c["d"], dtype=np.float32 if dt == "f32" else np.float64)
        return torch.from_numpy(xq).cuda()
    return S.queries_torch(c["d"], c["m"], c["seed"], device="cuda", dtype=tdt(torch, dt))


@pytest.mark.parametrize("cfg,source,k", CASES)
def test_evaluate_parity_configs(P, torch, oracle, cfg, source, k):
    c = S.CONFIGS[cfg]
    d, n, dt = c["d"], c["n"], c["dtype"]
    g = P.Grid(d, n)
    alpha = hierarchized_alpha(torch, P, g, source, dt, seed=c["seed"])
    x = config_queries(torch, cfg, dt)
    y = g.evaluate(alpha, x, presorted="plane" in c)
    torch.cuda.synchronize()
    m = x.shape[0]
    rng = np.random.default_rng(c["seed"] & 0xFFFF)
    samp = np.arange(m) if k is None or k >= m else np.sort(rng.choice(m, k, replace=False))
    xs = x.cpu().numpy()[samp].astype(np.float64)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), xs)
    check_eval(y.cpu().numpy()[samp], yo, ao, TOL[dt], f"{cfg}/{source}")
    if source != "B":  # positive surpluses: plain relative error too
        rel = np.abs(y.cpu().numpy()[samp] - yo) / np.abs(yo)
        assert rel.max() <= TOL[dt]


def separable_dp_torch(torch, d, n, X):
    """Pin P8 on the device: for function A the surpluses factor into 1D
    closed forms 4^-l (1 - c + 3 c x_centre), so
    f_s(x) = sum_{m<n} [z^m] prod_t sum_l a_t(l) z^l (layout-free, O(d n^2))."""
    c = (torch.arange(d, dtype=torch.float64, device=X.device) + 1.0) / (2.0 * d + 2.0)
    m = X.shape[0]
    poly = torch.zeros((m, n), dtype=torch.float64, device=X.device)
    poly[:, 0] = 1.0
    for t in range(d):
        xt = X[:, t].to(torch.float64)
        a = torch.zeros((m, n), dtype=torch.float64, device=X.device)
        for lev in range(n):
            k = torch.clamp(torch.floor(xt * 2.0 ** lev), 0, 2 ** lev - 1)
            centre = (2 * k + 1) / 2.0 ** (lev + 1)
            s = 4.0 ** -lev * (1.0 - c[t] + 3.0 * c[t] * centre)
            a[:, lev] = s * torch.clamp(1.0 - torch.abs(xt * 2.0 ** (lev + 1) - (2 * k + 1)), min=0.0)
        new = torch.zeros_like(poly)
        for p in range(n):
            new[:, p:] += poly[:, p:p + 1] * a[:, :n - p]
        poly = new
    return poly.sum(1)


def closed_form_alpha_A(torch, oracle, g, dt):
    """Exact (closed-form) surpluses of function A for every grid point (P5'), at the (l, i) of every index
    given by the ORACLE's idx2gp (pinned independently of libsg), computed on the device."""
    d = g.d
    c = (torch.arange(d, dtype=torch.float64, device="cuda") + 1.0) / (2.0 * d + 2.0)
    out = torch.empty(g.num_points, dtype=tdt(torch, dt), device="cuda")
    chunk = 1 << 23
    for a in range(0, g.num_points, chunk):
        b = min(g.num_points, a + chunk)
        lo, io = oracle.idx2gp(d, g.n, np.arange(a, b, dtype=np.uint64))
        l = torch.from_numpy(lo).cuda().to(torch.float64)
        x = torch.from_numpy(io).cuda().to(torch.float64) / torch.pow(2.0, l + 1.0)
        out[a:b] = torch.prod(torch.pow(4.0, -l) * (1.0 - c + 3.0 * c * x), dim=1).to(out.dtype)
    return out


def test_evaluate_cfg3_full_size(P, torch, oracle):
    """The bench workload (d=10, n=11, 10^7 queries, Morton-ordered inside
    sg_evaluate): a seeded sample against the oracle on the hierarchized
    surpluses, and ALL 10^7 outputs against the separable closed form."""
    c = S.CONFIGS["cfg3"]
    d, n, m = c["d"], c["n"], c["m"]
    g = P.Grid(d, n)
    x = S.queries_torch(d, m, c["seed"], device="cuda")
    alpha = hierarchized_alpha(torch, P, g, "A", "f64")
    y = g.evaluate(alpha, x)
    torch.cuda.synchronize()
    rng = np.random.default_rng(3)
    samp = np.sort(rng.choice(m, 10_000, replace=False))  # K = 10^4 oracle queries at cfg3
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy(), x[torch.from_numpy(samp).cuda()].cpu().numpy())
    check_eval(y.cpu().numpy()[samp], yo, ao, TOL["f64"], "cfg3 oracle sample")
    del alpha
    exact = closed_form_alpha_A(torch, oracle, g, "f64")
    y2 = g.evaluate(exact, x)
    worst = 0.0
    for a in range(0, m, 1 << 21):
        b = min(m, a + (1 << 21))
        ref = separable_dp_torch(torch, d, n, x[a:b])
        rel = ((y2[a:b] - ref).abs() / ref.abs()).max().item()
        worst = max(worst, rel)
    assert worst <= 1e-12, worst


def test_evaluate_cfg3_random_surplus_sample(P, torch, oracle):
    c = S.CONFIGS["cfg3"]
    d, n = c["d"], c["n"]
    g = P.Grid(d, n)
    alpha = S.random_surplus_torch(g.num_points, seed=99, device="cuda")
    x = S.queries_torch(d, 20000, 1234, device="cuda")
    y = g.evaluate(alpha, x)
    samp = np.arange(0, 20000, 2)  # 10^4 of the call's queries
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy(), x[torch.from_numpy(samp).cuda()].cpu().numpy())
    check_eval(y.cpu().numpy()[samp], yo, ao, TOL["f64"], "cfg3 source B")


# ----------------------------------------------------------------- edge cases
@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_evaluate_edge_cases(P, torch, oracle, dt):
    d, n = 3, 6
    g = P.Grid(d, n)
    alpha = hierarchized_alpha(torch, P, g, "B", dt, seed=4)
    T = tdt(torch, dt)
    # m = 0
    y0 = g.evaluate(alpha, torch.empty((0, d), dtype=T, device="cuda"))
    assert y0.numel() == 0
    # domain boundary, outside, NaN, grid points, cell boundaries, x = 1
    pts = np.array([[0.0, 0.5, 0.5], [1.0, 0.5, 0.5], [-0.25, 0.3, 0.3], [0.3, 1.5, 0.2], [np.nan, 0.2, 0.2],
                    [0.5, 0.25, 0.75], [0.125, 0.0625, 0.5], [1.0 - 2.0 ** -40, 0.5, 0.5],
                    [2.0 ** -30, 0.5, 0.5], [np.inf, 0.5, 0.5], [0.375, 0.625, 0.875]])
    x = torch.tensor(pts, dtype=T, device="cuda")
    y = g.evaluate(alpha, x).cpu().numpy().astype(np.float64)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), x.cpu().numpy().astype(np.float64))
    assert np.isnan(y[4]) and np.isnan(yo[4])
    ok = ~np.isnan(yo)
    assert np.all(y[[0, 1, 2, 3, 9]] == 0.0)
    check_eval(y[ok], yo[ok], ao[ok], TOL[dt], "edge")
    # interpolation at the grid points (P6): f_s(x_j) = sum over ancestors = nodal values
    xs = g.coords(dtype=T)
    yg = g.evaluate(alpha, xs).cpu().numpy().astype(np.float64)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), xs.cpu().numpy().astype(np.float64))
    check_eval(yg, yo, ao, TOL[dt], "grid points")


@pytest.mark.parametrize("d,n", [(5, 8), (20, 6), (10, 9)])
def test_evaluate_edge_cases_specialised(P, torch, oracle, d, n):
    """Edge cases through the specialised trie kernels (cfg2 d=5 n=8; cfg5 d=20
    n=6 with the level-0 suffix products and the budget-1 Horner pass, whose
    level-1 digit is taken from x >= 0.5; the cfg3 kernels at d=10 n=9, whose
    trie dimensions take their hats by doubling): dyadic coordinates (cell
    boundaries at every level), 0.5 exactly, 1 - 2^-40, tiny, and rows with
    one coordinate on / outside the boundary (value 0) or NaN."""
    g = P.Grid(d, n)
    alpha = hierarchized_alpha(torch, P, g, "B", "f64", seed=d)
    rng = np.random.default_rng(100 + d)
    pool = np.array([0.5, 0.25, 0.75, 1.0 / 64, 63.0 / 64, 2.0 ** -30, 1.0 - 2.0 ** -40, 0.375, 0.625])
    m = 48
    x = rng.random((m, d))
    special = rng.random((m, d)) < 0.6
    x[special] = rng.choice(pool, size=int(special.sum()))
    x[0, :] = 0.5
    bad = {1: 0.0, 2: 1.0, 3: -0.25, 4: 1.5, 5: np.inf}
    for r, v in bad.items():
        x[r, rng.integers(d)] = v
    x[6, d - 1] = np.nan
    last = {7: 1.0, 8: -0.25, 9: 1.5, 10: 0.0}  # the last dimension (a trie dimension: hats by doubling)
    for r, v in last.items():
        x[r, d - 1] = v
    xt = torch.tensor(x, dtype=torch.float64, device="cuda")
    y = g.evaluate(alpha, xt).cpu().numpy()
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy(), x)
    assert np.isnan(y[6]) and np.isnan(yo[6])
    assert np.all(y[list(bad) + list(last)] == 0.0)
    ok = ~np.isnan(yo)
    check_eval(y[ok], yo[ok], ao[ok], TOL["f64"], f"edge d={d}")


@pytest.mark.parametrize("m", [1, 31, 33, 1000, 4097])
def test_evaluate_ragged_sizes(P, torch, oracle, m):
    d, n = 5, 6
    g = P.Grid(d, n)
    alpha = hierarchized_alpha(torch, P, g, "B", "f64", seed=m)
    x = S.queries_torch(d, m, 1000 + m, device="cuda")
    y = g.evaluate(alpha, x).cpu().numpy()
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy(), x.cpu().numpy())
    check_eval(y, yo, ao, TOL["f64"], f"m={m}")


def test_presorted_host_and_partition_invariance(P, torch):
    """Per-query arithmetic order is fixed by the enumeration, so the result is
    bitwise independent of the query order, of the SFC pass, of the host-buffer
    entry point and of how the batch is split (multi-GPU partitions)."""
    c = S.CONFIGS["cfg2"]
    d, n = c["d"], c["n"]
    g = P.Grid(d, n)
    alpha = hierarchized_alpha(torch, P, g, "A", "f64")
    x = S.queries_torch(d, 200000, 77, device="cuda")
    y = g.evaluate(alpha, x)
    y_pre = g.evaluate(alpha, x, presorted=True)
    assert torch.equal(y, y_pre)
    perm = torch.randperm(x.shape[0], device="cuda")
    assert torch.equal(g.evaluate(alpha, x[perm])[torch.argsort(perm)], y)
    parts = torch.cat([g.evaluate(alpha, x[a:a + 50000]) for a in range(0, 200000, 50000)])
    assert torch.equal(parts, y)
    xh = x.cpu().pin_memory()
    yh = g.evaluate_host(alpha, xh)
    assert torch.equal(yh, y.cpu())
    ws = torch.empty(g.workspace_bytes(x.shape[0]), dtype=torch.uint8, device="cuda")
    assert torch.equal(g.evaluate(alpha, x, workspace=ws), y)


def test_evaluate_generic_kernel_matches(P, torch, oracle):
    """The generic fallback kernel (flag SG_EVAL_GENERIC) against the oracle."""
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    for cfg in ("cfg2", "cfg5"):
        c = S.CONFIGS[cfg]
        d, n = c["d"], c["n"]
        g = P.Grid(d, n)
        alpha = hierarchized_alpha(torch, P, g, "B", "f64", seed=7)
        x = S.queries_torch(d, 3000, 5, device="cuda")
        y = torch.empty(x.shape[0], dtype=torch.float64, device="cuda")
        _sg.sg_evaluate(g.handle, alpha, x, y, flags=_sg.SG_EVAL_GENERIC)
        samp = np.arange(0, 3000, 30)
        yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy(), x.cpu().numpy()[samp])
        check_eval(y.cpu().numpy()[samp], yo, ao, TOL["f64"], cfg + " generic")
