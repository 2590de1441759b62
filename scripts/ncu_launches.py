#!/usr/bin/env python
"""Aggregate an `ncu --metrics gpu__time_duration.sum --csv` launch list per kernel.

    python scripts/ncu_launches.py gpurun_out/X_launches.csv > profiles/X_launches.txt

ncu serialises launches and runs them cold, so the absolute times are not bench
numbers; the per-kernel SHARE of the step is what profiles/ records.
"""
import collections
import csv
import sys

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3}


def main(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        k = r[ki].split("(")[0]
        agg[k][0] += 1
        agg[k][1] += float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1.0)
    tot = sum(a[1] for a in agg.values())
    print(f"{'kernel':120s} {'launches':>8s} {'total ms':>12s} {'share':>7s}")
    for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{k[:120]:120s} {c:8d} {t:12.3f} {100 * t / tot:6.2f}%")


if __name__ == "__main__":
    main(sys.argv[1])
