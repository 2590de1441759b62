"""Host model of the support enumeration of csrc/exp/eval_sparse.cuh (cfg5 kernel), pinned to the oracle.

The kernel enumerates the level vectors of a group by their highest non-zero dimension u and its level v,
with the subspace offset off(u, B, v) = C(B+u, u) - C(B-v+u, u) and dimension u's cell digits at bit J - B.
This test re-runs that recursion in Python (the same formulas, no GPU) and checks, against the oracle's
Alg. 3 enumeration (or_enumerate) and gp2idx (Alg. 5), that it visits every level vector of the group exactly
once at its bijection rank, and that the index it forms for random cells is gp2idx's (Alg. 3 P:L373,
Alg. 5, index3 P:L381-L389).
"""
from math import comb

import numpy as np
import pytest

import oracle


def sparse_terms(d, j, cells):
    """[(rank, level vector, in-subspace index)] of group j, in the kernel's visiting order; cells[t][v] = k_t(v)."""
    out = []

    def G(t, B, b, P, lv):
        sh = j - B
        l0 = list(lv)
        l0[0] = B
        out.append((b, tuple(l0), P | (cells[0][B] << sh)))  # u = 0: l_1..l_t = 0, l_0 = B
        for u in range(1, t + 1):  # leaves: l_u = B
            l1 = list(lv)
            l1[u] = B
            out.append((b + comb(B + u, u) - 1, tuple(l1), P | (cells[u][B] << sh)))
        for v in range(1, B):  # internal nodes
            for u in range(1, t + 1):
                l2 = list(lv)
                l2[u] = v
                G(u - 1, B - v, b + comb(B + u, u) - comb(B - v + u, u), P | (cells[u][v] << sh), l2)

    if j == 0:
        return [(0, tuple([0] * d), 0)]
    G(d - 1, j, 0, 0, [0] * d)
    return out


@pytest.mark.parametrize("d,n", [(1, 4), (2, 5), (3, 4), (5, 5), (8, 4), (20, 6), (14, 6)])
def test_sparse_enumeration_matches_the_bijection(d, n):
    rng = np.random.default_rng(d * 10 + n)
    for j in range(n):
        ref = oracle.enumerate_group(d, j)
        x = rng.random(d)
        cells = [[int(min(np.floor(x[t] * 2 ** v), 2 ** v - 1)) for v in range(n)] for t in range(d)]
        terms = sparse_terms(d, j, cells)
        assert len(terms) == len(ref) == comb(j + d - 1, d - 1)
        ranks = sorted(r for r, _, _ in terms)
        assert ranks == list(range(len(ref))), "every subspace of the group exactly once"
        base = oracle.index3(d, j)
        r = np.array([t[0] for t in terms], dtype=np.uint64)
        L = np.array([t[1] for t in terms], dtype=np.int32)
        idx = np.array([t[2] for t in terms], dtype=np.uint64)
        assert np.array_equal(ref[r.astype(np.int64)], L), f"d={d} j={j}: level vectors at their ranks"
        c = np.array(cells, dtype=np.int32)  # [t][v]
        i = 2 * c[np.arange(d)[None, :], L] + 1
        g = oracle.gp2idx(L, i)
        assert np.array_equal(g, np.uint64(base) + (r << np.uint64(j)) + idx), f"d={d} j={j}"
