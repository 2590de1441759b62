#!/usr/bin/env python
"""Small calls through every libsg kernel family, for compute-sanitizer (memcheck / racecheck / initcheck).

    compute-sanitizer --tool racecheck python scripts/sanitize_run.py > profiles/rNN_racecheck.txt

Shapes are small so that the instrumented run finishes in minutes: the specialised tries (cfg1 d=2 n=3, d=5
n=6 on the d5n8 instantiation, d=10 n=5 on the cfg3 instantiation with its split launches, d=20 n=4 on the
S0 instantiation, fp32 d=3 n=8 on the cfg4 instantiation), the generic kernel (d=7 n=5, fp64 and fp32), the
fallback (SG_EVAL_GENERIC), the Morton sort, the index maps, coordinates, and the hierarchization (pole
families incl. n=14 fp64 with the shared-memory opt-in, and the global fallback at d=1 n=17).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import sginputs as S  # noqa: E402
import paper_conf_ppopp_murarasuwbbp11_b200 as P  # noqa: E402
from paper_conf_ppopp_murarasuwbbp11_b200 import _sg  # noqa: E402


def run(d, n, dt=torch.float64, m=700, generic=False):
    g = P.Grid(d, n)
    v = S.f_A_torch(g.coords()).to(dt)
    a = g.hierarchize_(v)
    x = S.queries_torch(d, m, 5 + d, device="cuda", dtype=dt)
    y = g.evaluate(a, x)
    if generic:
        _sg.sg_evaluate(g.handle, a, x, y, flags=_sg.SG_EVAL_GENERIC)
    perm = g.sfc_order(x)
    g.evaluate_ordered(a, x, perm, m // 7, m // 3, out=y)
    idx = torch.arange(min(g.num_points, 4096), dtype=torch.int64, device="cuda")
    l, i = g.idx2gp(idx)
    g.gp2idx(l, i)
    torch.cuda.synchronize()
    print(f"d={d} n={n} {dt}: ok, N={g.num_points}", flush=True)
    g.close()


if __name__ == "__main__":
    torch.cuda.set_device(0)
    run(2, 3)
    run(5, 6, generic=True)
    run(10, 5)
    run(20, 4)
    run(3, 8, torch.float32, m=1000)
    run(7, 5)
    run(7, 5, torch.float32, generic=True)
    run(3, 14, m=64)
    run(1, 17, m=64)
    # visualization slice, sharded-grid parts, boundary grid
    g = P.Grid(3, 8)
    a = g.hierarchize_(S.f_A_torch(g.coords()))
    g.render_plane(a, [0.0, 0.0, 0.3], [1 / 64, 0.0, 0.0], [0.0, 1 / 32, 0.0], 64, 32, order=1)
    x = S.queries_torch(3, 500, 3, device="cuda")
    y = torch.zeros(500, dtype=torch.float64, device="cuda")
    for r in range(3):
        first, count = g.part_bounds(3, r)
        g.evaluate_part(a[first:first + count].clone(), 3, r, x, out=y, accumulate=True)
    bg = P.BoundaryGrid(3, 4)
    ba = bg.hierarchize_(S.f_A_torch(bg.coords()) + 1.0)
    bg.evaluate(ba, x)
    torch.cuda.synchronize()
    print("plane / parts / boundary: ok", flush=True)
    print("sanitize run complete")
