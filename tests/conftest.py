import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


@pytest.fixture(scope="session")
def oracle():
    import oracle as O
    O.build()
    return O


def all_points_structural(d, n):
    """Independent construction of the layout described in Sec. 4.1:
    level groups by ascending |l|_1, subspaces of a group in Alg. 3 order (last
    component slowest, i.e. lexicographic on (l_{d-1}, ..., l_1)),
    points of a subspace in the order of Alg. 5 line 3 (C-order ravel, dimension 0
    most significant).  Returns (L, I) arrays of shape (N, d) in layout order."""
    import itertools
    Ls, Is = [], []
    for j in range(n):
        group = [l for l in itertools.product(range(j + 1), repeat=d) if sum(l) == j]
        group.sort(key=lambda l: tuple(reversed(l[1:])))
        for l in group:
            shape = tuple(1 << lt for lt in l)
            for cell in itertools.product(*[range(s) for s in shape]):  # C order
                Ls.append(l)
                Is.append(tuple(2 * k + 1 for k in cell))
    return np.array(Ls, dtype=np.int32).reshape(-1, d), np.array(Is, dtype=np.int32).reshape(-1, d)


def hat_np(level, index, x):
    """phi(2^{l+1} x - i), phi(y) = max(1 - |y|, 0)  (P:L87, 0-based levels)."""
    return np.maximum(1.0 - np.abs(np.ldexp(x, level + 1) - index), 0.0)


def gpu_available():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False
