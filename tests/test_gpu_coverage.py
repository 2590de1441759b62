"""GPU parity across the evaluation dispatch: every shape class libsg's sg_evaluate routes to a different
kernel (specialised trie kernels, the generic-shape kernel, the fallback) against the CPU oracle, in
both dtypes; d = 1 (the paper assumes d >= 2, reading G6) against the piecewise-linear
interpolant (pin P10); the multi-GPU building blocks (sg_sfc_order / sg_evaluate_ordered) against one
sg_evaluate call, bitwise (pin P12), including a world-size-2 gloo group on one GPU that runs
multi.evaluate_distributed with libsg's kernels.

Tolerance (reading G13): |y - y_oracle| <= tol * sum_terms |alpha phi|, tol 1e-12 (fp64), 1e-5 (fp32).
"""
import os
import socket

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


def check_eval(y, yo, ao, tol, what):
    y = np.asarray(y, dtype=np.float64)
    worst = float(np.max(np.abs(y - yo) / np.maximum(ao, np.finfo(float).tiny))) if y.size else 0.0
    assert worst <= tol, f"{what}: normwise error {worst:.3e} > {tol:.0e}"


def surpluses(torch, g, source, dt, seed):
    if source == "B":
        return S.random_surplus_torch(g.num_points, seed=seed, device="cuda", dtype=tdt(torch, dt))
    x = g.coords(dtype=torch.float64)
    v = S.f_A_torch(x).to(tdt(torch, dt))
    return g.hierarchize_(v)


# (d, n): one case per dispatch class of sg_evaluate (DESIGN.md 6.1 "Dispatch"), plus off-benchmark shapes
SHAPES = [(1, 1), (1, 6), (1, 11), (2, 2), (2, 3), (2, 9), (3, 5), (3, 10), (3, 14), (4, 7), (5, 3), (5, 8),
          (5, 9), (5, 10), (5, 11), (6, 6), (7, 5), (8, 6), (9, 4), (10, 3), (10, 6), (10, 9), (11, 5), (12, 4),
          (12, 6), (16, 4), (20, 3), (20, 5), (20, 6), (32, 3)]


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("d,n", SHAPES)
def test_evaluate_shapes_vs_oracle(P, torch, oracle, d, n, dt):
    g = P.Grid(d, n)
    for source, seed in (("A", 0), ("B", 1000 * d + n)):
        alpha = surpluses(torch, g, source, dt, seed)
        x = S.queries_torch(d, 1537, 77 + d * 31 + n, device="cuda", dtype=tdt(torch, dt))
        y = g.evaluate(alpha, x).cpu().numpy()
        k = 1537 if d * n <= 60 else 300
        samp = np.linspace(0, 1536, k).astype(np.int64)
        yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64),
                                 x.cpu().numpy()[samp].astype(np.float64))
        check_eval(y[samp], yo, ao, TOL[dt], f"d={d} n={n} {dt} source {source}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("d,n", [(2, 3), (5, 8), (10, 5), (20, 4)])
def test_generic_fallback_kernel(P, torch, oracle, d, n, dt):
    """The unspecialised kernel (flag SG_EVAL_GENERIC) in both dtypes."""
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    g = P.Grid(d, n)
    alpha = surpluses(torch, g, "B", dt, 7)
    x = S.queries_torch(d, 700, 5, device="cuda", dtype=tdt(torch, dt))
    y = torch.empty(x.shape[0], dtype=x.dtype, device="cuda")
    _sg.sg_evaluate(g.handle, alpha, x, y, flags=_sg.SG_EVAL_GENERIC)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), x.cpu().numpy().astype(np.float64))
    check_eval(y.cpu().numpy(), yo, ao, TOL[dt], f"generic d={d} n={n} {dt}")


@pytest.mark.parametrize("n", [1, 6, 11])
def test_d1_piecewise_linear_interpolant(P, torch, n):
    """Pin P10 on the GPU: in one dimension the sparse grid is the full grid of mesh 2^-n, so f_s is the
    piecewise-linear interpolant of the nodal values (numpy.interp) -- independent of the layout."""
    g = P.Grid(1, n)
    xs = g.coords().cpu().numpy()[:, 0]
    f = lambda t: np.sin(5.0 * t) * t * (1.0 - t) + 0.3 * t * (1.0 - t)  # zero on the boundary
    v = torch.from_numpy(f(xs)).cuda()
    alpha = g.hierarchize_(v.clone())
    q = np.concatenate([S.queries(1, 4000, 99)[:, 0], np.sort(xs), [0.0, 1.0, -0.5, 1.5]])
    y = g.evaluate(alpha, torch.from_numpy(q[:, None]).cuda()).cpu().numpy()
    knots = np.concatenate([[0.0], np.sort(xs), [1.0]])
    vals = np.concatenate([[0.0], f(np.sort(xs)), [0.0]])
    ref = np.where((q >= 0) & (q <= 1), np.interp(q, knots, vals), 0.0)
    np.testing.assert_allclose(y, ref, rtol=0, atol=16 * n * np.finfo(float).eps * max(1.0, np.abs(vals).max()))


def test_fp32_cfg4_plane_edge_cases(P, torch, oracle):
    """fp32 d=3 n=14 (the cfg4 kernel): cell boundaries at every level, the plane's x2, 0.5, tiny, and
    coordinates on / outside the boundary and NaN."""
    d, n = 3, 14
    g = P.Grid(d, n)
    alpha = surpluses(torch, g, "B", "f32", 4)
    rng = np.random.default_rng(314)
    pool = np.array([0.5, 0.25, 0.75, 0.3, 1.0 / 8192, 8191.0 / 8192, 2.0 ** -20, 1.0 - 2.0 ** -20, 0.375],
                    dtype=np.float32)
    m = 64
    x = rng.random((m, d)).astype(np.float32)
    special = rng.random((m, d)) < 0.6
    x[special] = rng.choice(pool, size=int(special.sum()))
    bad = {1: 0.0, 2: 1.0, 3: -0.25, 4: 1.5, 5: np.inf}
    for r, v in bad.items():
        x[r, rng.integers(d)] = v
    x[6, 2] = np.nan
    xt = torch.from_numpy(x).cuda()
    for presorted in (False, True):
        y = g.evaluate(alpha, xt, presorted=presorted).cpu().numpy().astype(np.float64)
        yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), x.astype(np.float64))
        assert np.isnan(y[6]) and np.isnan(yo[6])
        assert np.all(y[list(bad)] == 0.0)
        ok = ~np.isnan(yo)
        check_eval(y[ok], yo[ok], ao[ok], TOL["f32"], f"cfg4 edge presorted={presorted}")


@pytest.mark.parametrize("cfg", ["cfg2", "cfg5"])
def test_ordered_ranges_bitwise_equal_one_call(P, torch, cfg):
    """Pin P12 with libsg's kernels: the P = 2, 4, 8 contiguous ranges of one sg_sfc_order permutation,
    evaluated one after the other with sg_evaluate_ordered, reproduce one sg_evaluate call bitwise;
    the order is deterministic (two calls agree) and a permutation."""
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    c = S.CONFIGS[cfg]
    g = P.Grid(c["d"], c["n"])
    alpha = surpluses(torch, g, "A", "f64", 0)
    x = S.queries_torch(c["d"], 100_003, 11, device="cuda")
    y_one = g.evaluate(alpha, x)
    perm = g.sfc_order(x)
    assert torch.equal(perm, g.sfc_order(x))
    assert torch.equal(torch.sort(perm.long()).values, torch.arange(x.shape[0], device="cuda"))
    for world in (2, 4, 8):
        y = torch.full_like(y_one, float("nan"))
        for r in range(world):
            first, count = multi.partition(x.shape[0], world, r)
            g.evaluate_ordered(alpha, x, perm, first, count, out=y)
        assert torch.equal(y, y_one), f"P={world}"
    # no order given: the batch taken as presorted, rows first..first+count-1
    y = torch.full_like(y_one, float("nan"))
    for r in range(3):
        first, count = multi.partition(x.shape[0], 3, r)
        g.evaluate_ordered(alpha, x, None, first, count, out=y)
    assert torch.equal(y, g.evaluate(alpha, x, presorted=True))


def test_evaluate_ordered_rejects_bad_range(P, torch):
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    g = P.Grid(3, 4)
    alpha = torch.zeros(g.num_points, dtype=torch.float64, device="cuda")
    x = torch.rand(10, 3, dtype=torch.float64, device="cuda")
    with pytest.raises(_sg.SgError):
        g.evaluate_ordered(alpha, x, None, 8, 5)
    with pytest.raises(ValueError):
        g.evaluate(alpha[:-1], x)
    with pytest.raises(ValueError):
        g.evaluate(alpha, x, out=torch.empty(10, dtype=torch.float32, device="cuda"))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _gloo_worker(rank, world, port, outdir):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_murarasuwbbp11_b200 as P
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        c = S.CONFIGS["cfg2"]
        g = P.Grid(c["d"], c["n"])
        alpha = torch.zeros(g.num_points, dtype=torch.float64, device="cuda")
        if rank == 0:
            alpha.copy_(g.hierarchize_(S.f_A_torch(g.coords())))
        x = S.queries_torch(c["d"], 50_001, 21, device="cuda")
        y, perm, first, count = multi.evaluate_distributed(g, alpha, x)  # broadcast + order + own range
        torch.cuda.synchronize()
        np.save(os.path.join(outdir, f"y{rank}.npy"), y.cpu().numpy())
        np.save(os.path.join(outdir, f"own{rank}.npy"), perm[first:first + count].cpu().numpy())
        if rank == 0:
            np.save(os.path.join(outdir, "ref.npy"), g.evaluate(alpha, x).cpu().numpy())
    finally:
        dist.destroy_process_group()


def test_gloo_world2_evaluate_distributed_on_one_gpu(tmp_path):
    """multi.evaluate_distributed with libsg's kernels on two ranks (gloo; both on cuda:0): the broadcast
    replicates rank 0's surpluses, the ranks agree on the order, and the assembled shards equal one
    sg_evaluate call bitwise."""
    import torch.multiprocessing as mp
    world = 2
    mp.spawn(_gloo_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    ref = np.load(tmp_path / "ref.npy")
    assembled = np.full(ref.shape, np.nan)
    owned = []
    for r in range(world):
        y = np.load(tmp_path / f"y{r}.npy")
        own = np.load(tmp_path / f"own{r}.npy")
        owned.append(own)
        assembled[own] = y[own]
    assert sorted(np.concatenate(owned).tolist()) == list(range(ref.size))
    assert np.array_equal(assembled, ref)


# ----------------------------------------------------------------- visualization slice (NEXT-3)
def plane_points(d, w, h, o, u, v, dtype):
    a = np.arange(w, dtype=np.float64) + 0.5
    b = np.arange(h, dtype=np.float64) + 0.5
    x = (o[None, None, :] + a[None, :, None] * u[None, None, :]) + b[:, None, None] * v[None, None, :]
    return x.reshape(h * w, d).astype(dtype)


@pytest.mark.parametrize("d,n,dt,w,h", [(3, 14, "f32", 256, 128), (3, 8, "f64", 64, 36), (5, 6, "f64", 40, 20),
                                        (10, 5, "f64", 33, 7), (2, 9, "f32", 16, 8)])
def test_render_plane_equals_evaluate(P, torch, oracle, d, n, dt, w, h):
    """sg_evaluate_plane: every pixel bitwise equal to sg_evaluate at the same point (row-major and
    Morton-tiled visiting orders), and a sample of pixels against the oracle."""
    g = P.Grid(d, n)
    alpha = surpluses(torch, g, "A", dt, 0)
    rng = np.random.default_rng(d * 100 + n)
    if d == 3 and n == 14:  # the cfg4 plane (reading G19), scaled down
        o, u, v = np.array([0.0, 0.0, 0.3]), np.array([1.0 / w, 0.0, 0.0]), np.array([0.0, 1.0 / h, 0.0])
    else:  # an oblique slice, partly outside the cube
        o = rng.random(d) * 0.3
        u = (rng.random(d) - 0.3) / w
        v = (rng.random(d) - 0.3) / h
    npdt = np.float32 if dt == "f32" else np.float64
    pts = torch.from_numpy(plane_points(d, w, h, o, u, v, npdt)).cuda()
    ref = g.evaluate(alpha, pts, presorted=True).reshape(h, w)
    for order in (0, 1):
        img = g.render_plane(alpha, o, u, v, w, h, order=order)
        assert torch.equal(img, ref), f"order {order}"
    k = np.linspace(0, w * h - 1, 200).astype(np.int64)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), pts.cpu().numpy()[k].astype(np.float64))
    check_eval(ref.reshape(-1).cpu().numpy()[k], yo, ao, TOL[dt], f"plane d={d} n={n}")


# ----------------------------------------------------------------- sharded grids (NEXT-4)
@pytest.mark.parametrize("d,n,parts,dt", [(3, 7, 3, "f64"), (6, 6, 4, "f64"), (10, 8, 8, "f64"), (10, 11, 2, "f64"),
                                          (12, 5, 5, "f64"), (7, 5, 40, "f64"), (3, 7, 3, "f32"), (6, 6, 4, "f32")])
def test_evaluate_parts_sum_to_the_grid(P, torch, oracle, d, n, parts, dt):
    """The parts of sg_part_bounds tile the layout exactly (contiguous, in order); each part evaluated from
    ONLY its own surpluses (a copy of its slice) sums to the whole-grid evaluation within the normwise
    tolerance, and a sample agrees with the oracle."""
    g = P.Grid(d, n)
    alpha = surpluses(torch, g, "B", dt, d + n)
    m = 20_000 if g.num_points < 5e7 else 2_000
    x = S.queries_torch(d, m, 31 * d + n, device="cuda", dtype=tdt(torch, dt))
    bounds = [g.part_bounds(parts, r) for r in range(parts)]
    pos = 0
    for first, count in bounds:
        assert first == pos or count == 0
        pos = first + count if count else pos
    assert pos == g.num_points
    y = torch.zeros(m, dtype=x.dtype, device="cuda")
    for r, (first, count) in enumerate(bounds):
        part = alpha[first:first + count].clone()  # the part's surpluses only
        g.evaluate_part(part, parts, r, x, out=y, accumulate=True)
    ref = g.evaluate(alpha, x)
    k = np.linspace(0, m - 1, 64).astype(np.int64)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), x.cpu().numpy()[k].astype(np.float64))
    check_eval(y.cpu().numpy()[k], yo, ao, TOL[dt], f"parts d={d} n={n} P={parts} {dt}")
    # whole batch against the one-call result: normwise with the oracle's A(x) scale bound |y| <= A
    # (fp32: each part's result is rounded to fp32 before the next part accumulates onto it)
    err = (y.double() - ref.double()).abs().max().item()
    assert err <= TOL[dt] * float(np.max(ao)) * 10 * (parts if dt == "f32" else 1), err


def _shard_worker(rank, world, port, outdir):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_murarasuwbbp11_b200 as P
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        g = P.Grid(8, 7)
        alpha = g.hierarchize_(S.f_A_torch(g.coords()))  # (every rank computes it here; it keeps only its part)
        first, count = g.part_bounds(world, rank)
        mine = alpha[first:first + count].clone()
        del alpha
        x = S.queries_torch(8, 30_001, 77, device="cuda")
        y = multi.evaluate_sharded_grid(g, mine, x)  # own part + one all-reduce
        torch.cuda.synchronize()
        np.save(os.path.join(outdir, f"y{rank}.npy"), y.cpu().numpy())
    finally:
        dist.destroy_process_group()


def test_gloo_world2_sharded_grid_on_one_gpu(P, torch, tmp_path):
    import torch.multiprocessing as mp
    world = 2
    mp.spawn(_shard_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    g = P.Grid(8, 7)
    alpha = g.hierarchize_(S.f_A_torch(g.coords()))
    ref = g.evaluate(alpha, S.queries_torch(8, 30_001, 77, device="cuda")).cpu().numpy()
    y0, y1 = np.load(tmp_path / "y0.npy"), np.load(tmp_path / "y1.npy")
    assert np.array_equal(y0, y1)  # every rank holds the reduced result
    np.testing.assert_allclose(y0, ref, rtol=1e-12, atol=0)  # positive surpluses: plain relative error


# ----------------------------------------------------------------- non-zero boundary (NEXT-2)
@pytest.mark.parametrize("d,n,dt", [(1, 5, "f64"), (2, 4, "f64"), (3, 3, "f64"), (3, 5, "f64"), (4, 3, "f64"),
                                    (2, 6, "f32")])
def test_boundary_grid_vs_oracle(P, torch, oracle, d, n, dt):
    """BoundaryGrid (sg_bcreate / sg_bcoords_device / sg_bhierarchize / sg_bevaluate) against the pinned
    boundary oracle: layout and coordinates exact, surpluses bit-exact (fp64), evaluations within the
    normwise tolerance at random points, grid points, boundary points and outside the cube."""
    from oracle import boundary as OB
    g = P.BoundaryGrid(d, n)
    assert g.num_points == OB.num_points(d, n)
    xp, _, _, _ = OB.points(d, n)
    for f, (S_, c) in enumerate(OB.faces(d)):
        fc = g.face(f)
        assert fc["free"] == list(S_)
        assert fc["fixed_bits"] == sum(b << k for k, b in enumerate(c))
    T = tdt(torch, dt)
    x = g.coords(dtype=T)
    np.testing.assert_array_equal(x.cpu().numpy().astype(np.float64), xp)
    f = np.sin(3.0 * xp.sum(1)) + 0.5 * xp[:, 0] * (1.0 - 0.3 * xp[:, -1]) + 0.25
    vals = torch.from_numpy(f).to(T).cuda()
    alpha = g.hierarchize_(vals.clone())
    want = OB.hierarchize(d, n, vals.cpu().numpy().astype(np.float64))
    if dt == "f64":
        np.testing.assert_array_equal(alpha.cpu().numpy(), want)
    else:
        np.testing.assert_allclose(alpha.cpu().numpy(), want, rtol=0, atol=1e-5 * np.abs(want).max() * d * n)
    q = np.concatenate([S.queries(d, 300, 17 + d), xp[:: max(1, len(xp) // 50)],
                        np.full((1, d), 0.0), np.full((1, d), 1.0), np.full((1, d), 1.5)])
    qt = torch.from_numpy(q).to(T).cuda()
    y = g.evaluate(alpha, qt).cpu().numpy().astype(np.float64)
    yo, ao = OB.evaluate(d, n, alpha.cpu().numpy().astype(np.float64), qt.cpu().numpy().astype(np.float64))
    check_eval(y, yo, ao, TOL[dt], f"boundary d={d} n={n} {dt}")
    assert y[-1] == 0.0  # outside the cube


def test_boundary_grid_reproduces_multilinear(P, torch):
    """The boundary basis spans the multilinear functions: f_s = f everywhere for f = prod (a_t + b_t x_t)."""
    d, n = 3, 5
    g = P.BoundaryGrid(d, n)
    a = torch.tensor([1.0, 0.5, 2.0], dtype=torch.float64, device="cuda")
    b = torch.tensor([0.3, -0.2, 1.1], dtype=torch.float64, device="cuda")
    ml = lambda z: torch.prod(a + b * z, dim=1)
    alpha = g.hierarchize_(ml(g.coords()))
    q = S.queries_torch(d, 5000, 9, device="cuda")
    torch.testing.assert_close(g.evaluate(alpha, q), ml(q), rtol=1e-13, atol=1e-14)
