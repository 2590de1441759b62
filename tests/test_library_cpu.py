"""CPU-side tests of the C-ABI library (no GPU needed): it loads, exports every
entry point include/sg.h declares, carries sm_100a code, and its host index maps
(sg_gp2idx / sg_idx2gp, Alg. 5 and inverse) are bit-exact against the oracle."""
import os
import re
import subprocess

import numpy as np
import pytest

from conftest import ROOT, gpu_available

HEADER = os.path.join(ROOT, "include", "sg.h")


@pytest.fixture(scope="module")
def P():
    from paper_conf_ppopp_murarasuwbbp11_b200 import build
    build.build()
    import paper_conf_ppopp_murarasuwbbp11_b200 as P
    return P


def declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sg_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    names = declared_symbols()
    for need in ("sg_create", "sg_gp2idx", "sg_idx2gp", "sg_hierarchize", "sg_evaluate"):
        assert need in names


def test_library_exports_every_declared_symbol(P):
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    out = subprocess.run(["nm", "-D", "--defined-only", _sg.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (sg_\w+)", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing
    assert set(_sg.EXPORTS) == set(declared_symbols())


def test_library_is_sm100a(P):
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    assert "sm_100a" in P.sg_build_info()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _sg.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


@pytest.mark.parametrize("d,n", [(1, 6), (2, 4), (3, 5), (5, 4), (10, 3), (20, 3), (32, 2)])
def test_host_maps_bit_exact_vs_oracle(P, oracle, d, n):
    h, N = P.sg_create(d, n)
    try:
        assert N == oracle.num_points(d, n)
        lay = P.sg_get_layout(h)
        assert lay["group_offset"] == [oracle.index3(d, j) for j in range(n + 1)]
        assert lay["group_count"] == [oracle.group_count(d, j) for j in range(n)]
        idx = np.arange(N, dtype=np.uint64)
        l, i = P.sg_idx2gp(h, idx, d)
        lo, io = oracle.idx2gp(d, n, idx)
        np.testing.assert_array_equal(l, lo)
        np.testing.assert_array_equal(i, io)
        np.testing.assert_array_equal(P.sg_gp2idx(h, lo, io), idx)
    finally:
        P.sg_destroy(h)


def test_host_maps_cfg3_sample(P, oracle):
    d, n = 10, 11
    h, N = P.sg_create(d, n)
    try:
        assert N == 127574017
        rng = np.random.default_rng(11)
        idx = np.concatenate([rng.integers(0, N, 100000, dtype=np.uint64), np.array([0, 1, N - 1], np.uint64)])
        l, i = P.sg_idx2gp(h, idx, d)
        lo, io = oracle.idx2gp(d, n, idx)
        np.testing.assert_array_equal(l, lo)
        np.testing.assert_array_equal(i, io)
        np.testing.assert_array_equal(P.sg_gp2idx(h, l, i), idx)
    finally:
        P.sg_destroy(h)


def test_host_maps_sentinels(P):
    h, N = P.sg_create(3, 4)
    try:
        with pytest.raises(P.SgError) as e:
            P.sg_idx2gp(h, np.array([0, N], np.uint64), 3)
        assert "SG_ERR_RANGE" in str(e.value)
        with pytest.raises(P.SgError):  # |l|_1 > n-1, even index, index out of range
            P.sg_gp2idx(h, [[2, 2, 0]], [[1, 1, 1]])
        from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
        import ctypes
        l = np.array([[0, 0, 0], [1, 0, 0], [0, 0, 1], [0, 0, 0]], np.int32)
        i = np.array([[1, 1, 1], [2, 1, 1], [1, 1, 5], [1, 1, 1]], np.int32)
        out = np.zeros(4, np.uint64)
        st = _sg.lib.sg_gp2idx(h, l.ctypes.data_as(ctypes.c_void_p), i.ctypes.data_as(ctypes.c_void_p), 4,
                               out.ctypes.data_as(ctypes.c_void_p))
        assert st == _sg.SG_ERR_RANGE
        np.testing.assert_array_equal(out, [0, 2 ** 64 - 1, 2 ** 64 - 1, 0])
    finally:
        P.sg_destroy(h)


def test_create_rejects_bad_args(P):
    for d, n in [(0, 3), (33, 2), (3, 0), (3, 32)]:
        with pytest.raises(P.SgError):
            P.sg_create(d, n)


@pytest.mark.skipif(gpu_available(), reason="checks the host-only handle")
def test_device_calls_without_gpu_fail_loudly(P):
    import ctypes
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    h, _ = P.sg_create(3, 4)
    try:
        st = _sg.lib.sg_evaluate(h, ctypes.c_void_p(8), ctypes.c_void_p(8), 1, ctypes.c_void_p(8), 0, 0, None, 0,
                                 None)
        assert st == _sg.SG_ERR_NODEV
        assert _sg.lib.sg_hierarchize(h, ctypes.c_void_p(8), 0, None) == _sg.SG_ERR_NODEV
    finally:
        P.sg_destroy(h)


def test_budget1_hat_ratio_reading():
    """DESIGN.md 6.1 (cfg5 budget-1 sub-tries): the d = 20 kernel sums a
    budget-1 sub-trie as S0[t] * sum_u alpha_u rho_u with rho = phi_1 / phi_0,
    which relies on (i) 0 <= phi_1(x) <= 2 phi_0(x) on [0, 1] (bounded,
    well-conditioned quotient) and (ii) phi_1 = 0 wherever phi_0 = 0.  Hat
    functions from P:L87, phi_{l,i}(x) = max(0, 1 - |2^{l+1} x - i|), level l
    having the odd indices i = 1, 3, .., 2^{l+1} - 1 (0-based levels)."""
    def phi(l, x):  # the one non-zero hat of level l at x (max over the level's cells)
        i = np.arange(1, 2 ** (l + 1), 2)[None, :]
        return np.max(np.maximum(0.0, 1.0 - np.abs(2.0 ** (l + 1) * x[:, None] - i)), axis=1)

    x = np.concatenate([np.linspace(-0.5, 1.5, 200001), np.arange(0, 65) / 64.0, [2.0 ** -40, 1 - 2.0 ** -40]])
    f0, f1 = phi(0, x), phi(1, x)
    assert np.all(f1 <= 2.0 * f0 + 1e-15)
    assert np.all(f1[f0 == 0.0] == 0.0)
    inside = (x > 0) & (x <= 0.25)
    np.testing.assert_allclose(f1[inside] / f0[inside], 2.0, rtol=1e-12)
    # the level-1 cell the kernel stores in the sign bit: k(1) = 1 iff x >= 1/2
    for xv in [0.25, 0.49999999, 0.5, 0.75, 1.0 - 2.0 ** -40]:
        k = int(np.clip(np.floor(2.0 * xv), 0, 1))
        assert k == (1 if xv >= 0.5 else 0)


@pytest.mark.parametrize("d,n", [(1, 6), (3, 7), (5, 4), (6, 6), (10, 11), (12, 5)])
def test_part_bounds_tile_the_layout(P, oracle, d, n):
    """sg_part_bounds (sharded grids, NEXT-4): P parts are contiguous, in layout order, cover [0, N) exactly,
    start at (group, l_{d-1}) boundaries (whole groups for d <= 5), and balance the subspace count."""
    h, N = P.sg_create(d, n)
    try:
        for parts in (1, 2, 3, 8):
            pos, subs = 0, []
            for r in range(parts):
                first, count = P.sg_part_bounds(h, parts, r)
                if count == 0:
                    subs.append(0)
                    continue
                assert first == pos
                pos = first + count
                # the part starts at a unit boundary: the point at `first` has its own subspace's first cell
                # and (for d <= 5) level sum = a group start
                l, i = oracle.idx2gp(d, n, np.array([first], dtype=np.uint64))
                assert np.all(i == 1)
                if d <= 5:
                    assert first in [oracle.index3(d, j) for j in range(n)]
                # subspaces in the part
                ls, _ = oracle.idx2gp(d, n, np.arange(first, first + count, dtype=np.uint64))
                subs.append(len({tuple(r_) for r_ in ls}) if count < 2_000_000 else None)
            assert pos == N
            T = oracle.binom(n - 1 + d, d)
            if parts > 1 and all(s is not None for s in subs) and d >= 6:
                unit = oracle.binom(n - 1 + d - 2, d - 2)  # the largest (group, l_{d-1}) unit
                assert sum(subs) == T and max(subs) <= -(-T // parts) + unit
    finally:
        P.sg_destroy(h)
