#!/usr/bin/env python
"""Time one config's sg_evaluate and check a sample against the oracle (experiment A/B helper).

    SG_LIB=paper_conf_ppopp_murarasuwbbp11_b200/libsg_exp.so SG_EXP_VAR=SP20 python scripts/exp_check.py cfg5

Prints one JSON line: evals/s (median of --reps device-timed calls after 2 warm-ups, CUDA events on the
current stream), the normwise error of --sample queries against oracle.evaluate, and the variant.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import sginputs as S  # noqa: E402
import paper_conf_ppopp_murarasuwbbp11_b200 as P  # noqa: E402

CFG = {"cfg2": (5, 8, 1_000_000), "cfg2p": (5, 10, 1_000_000), "cfg3": (10, 11, 10_000_000),
       "cfg5": (20, 6, 1_000_000), "d16n5": (16, 5, 1_000_000), "d14n6": (14, 6, 1_000_000),
       "d11n10": (11, 10, 2_000_000), "d12n9": (12, 9, 2_000_000), "d8n11": (8, 11, 2_000_000),
       "d6n12": (6, 12, 2_000_000)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--sample", type=int, default=300)
    a = ap.parse_args()
    d, n, m = CFG[a.cfg]
    g = P.Grid(d, n)
    v = S.f_A_torch(g.coords())
    alpha = g.hierarchize_(v)
    x = S.queries_torch(d, m, 0x5EED0005, device="cuda")
    y = torch.empty(m, dtype=torch.float64, device="cuda")
    ws = torch.empty(g.workspace_bytes(m), dtype=torch.uint8, device="cuda")
    fn = lambda: g.evaluate(alpha, x, out=y, workspace=ws)  # noqa: E731
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.reps)]
    for e0, e1 in ev:
        e0.record()
        fn()
        e1.record()
    torch.cuda.synchronize()
    ms = statistics.median(e0.elapsed_time(e1) for e0, e1 in ev)
    k = np.linspace(0, m - 1, a.sample).astype(np.int64)
    yo, ao = oracle.evaluate(d, n, alpha.cpu().numpy(), x.cpu().numpy()[k])
    err = float(np.max(np.abs(y.cpu().numpy()[k] - yo) / ao))
    print(json.dumps({"cfg": a.cfg, "var": os.environ.get("SG_EXP_VAR", "-"), "evals_per_s": m / (ms / 1e3),
                      "ms": ms, "normwise_err": err, "pass": err <= 1e-12}))


if __name__ == "__main__":
    main()
