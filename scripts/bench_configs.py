#!/usr/bin/env python
"""Device-timed sg_evaluate / sg_hierarchize throughput for every BASELINE.json config (1 GPU).

    python scripts/bench_configs.py [--reps 5] [--only cfg3,cfg5] > profiles/rNN_configs.txt
    python scripts/bench_configs.py --sweep [--reps 3] > profiles/rNN_sweep.txt

Per config: evaluations/s of sg_evaluate (Morton ordering + evaluation kernels
+ scatter, CUDA events around the call on the current stream, median of
--reps after 2 warm-ups), the fraction of the ideal L1 gather roofline
(T fp64/fp32 words per query at 128 B/clk/SM x 148 SMs x sm_max_mhz, DESIGN.md
6.1) and hierarchized points/s.  Inputs are the seeded recipes of sginputs/
(function A surpluses).  SURVEY.md 8(d): "all configs at 1 GPU".
"""
import json
import math
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import sginputs as S  # noqa: E402
import paper_conf_ppopp_murarasuwbbp11_b200 as P  # noqa: E402


def timed(fn, reps):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    for a, b in ev:
        a.record()
        fn()
        b.record()
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) for a, b in ev)


def sweep(reps, f_mhz):
    """Per-term throughput of sg_evaluate for every d in [1,12], n in [2,12] (random surpluses, source B;
    10^6 queries, fewer for the largest grids): which kernel serves a shape must not cost more than ~2x
    of the cfg3 per-term rate."""
    for d in range(1, 13):
        for n in range(2, 13):
            g = P.Grid(d, n)
            N, T = g.num_points, g.num_subspaces
            if N >= (1 << 31) or N * 8 > 20e9:
                g.close()
                continue
            m = 1_000_000 if T <= 20_000 else (1 << 18 if T <= 400_000 else 1 << 16)
            alpha = S.random_surplus_torch(N, seed=7, device="cuda")
            x = S.queries_torch(d, m, 1234 + d, device="cuda")
            y = torch.empty(m, dtype=torch.float64, device="cuda")
            ws = torch.empty(g.workspace_bytes(m), dtype=torch.uint8, device="cuda")
            ms = timed(lambda: g.evaluate(alpha, x, out=y, workspace=ws), reps)
            rate = m / (ms / 1e3)
            print(json.dumps({"d": d, "n": n, "points": N, "terms": T, "queries": m, "evaluate_ms": round(ms, 3),
                              "evals_per_s": rate, "terms_per_s": rate * T,
                              "gather_roofline_frac": round(rate * T * 8 / (148 * 128 * f_mhz * 1e6), 4)}), flush=True)
            g.close()
            del alpha, x, y, ws
            torch.cuda.empty_cache()


def main():
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 5
    pk_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    f_mhz = json.load(open(pk_path)).get("sm_max_mhz", 1965.0) if os.path.exists(pk_path) else 1965.0
    torch.cuda.set_device(0)
    if "--sweep" in sys.argv:
        return sweep(reps, f_mhz)
    names = ["cfg1", "cfg2", "cfg2p", "cfg3", "cfg4", "cfg5"]
    if "--only" in sys.argv:
        names = sys.argv[sys.argv.index("--only") + 1].split(",")
    for name in names:
        c = S.CONFIGS[name]
        d, n = c["d"], c["n"]
        dt = torch.float32 if c["dtype"] == "f32" else torch.float64
        g = P.Grid(d, n)
        vals = torch.empty(g.num_points, dtype=torch.float64, device="cuda")
        for a in range(0, g.num_points, 1 << 23):
            b = min(g.num_points, a + (1 << 23))
            vals[a:b] = S.f_A_torch(g.coords(a, b - a))
        vals = vals.to(dt)
        alpha = vals.clone()
        # hierarchization is in place: time (restore the nodal values + hierarchize) minus the restore
        hier_ms = timed(lambda: (alpha.copy_(vals), g.hierarchize_(alpha)), reps) - timed(lambda: alpha.copy_(vals), reps)
        presorted = "plane" in c
        if presorted:
            w, h, x2 = c["plane"]
            x = torch.from_numpy(S.plane_queries(w, h, x2, d=d, dtype=np.float32 if dt == torch.float32
                                                 else np.float64)).cuda()
        else:
            x = S.queries_torch(d, c["m"], c["seed"], device="cuda", dtype=dt)
        m = x.shape[0]
        y = torch.empty(m, dtype=dt, device="cuda")
        ws = torch.empty(g.workspace_bytes(m, dt, presorted), dtype=torch.uint8, device="cuda")
        ev_ms = timed(lambda: g.evaluate(alpha, x, out=y, presorted=presorted, workspace=ws), reps)
        T = g.num_subspaces
        word = 4 if dt == torch.float32 else 8
        rate = m / (ev_ms / 1e3)
        lsu_peak = 148 * 128 * f_mhz * 1e6  # B/s
        frac = rate * T * word / lsu_peak
        fma = math.comb(n + d, d) - 1
        print(json.dumps({"config": name, "d": d, "n": n, "dtype": c["dtype"], "points": g.num_points,
                          "queries": m, "presorted": presorted, "evaluate_ms": round(ev_ms, 3),
                          "evals_per_s": rate, "gather_roofline_frac": round(frac, 4),
                          "fp64_or_fp32_tflops": 2 * fma * rate / 1e12,
                          "hierarchize_ms": round(hier_ms, 3),
                          "hierarchized_points_per_s": g.num_points / (hier_ms / 1e3)}), flush=True)
        g.close()
        del alpha, vals, x, y, ws
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
