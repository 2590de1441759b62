#!/usr/bin/env python
"""DRAM traffic of one sg_evaluate call (all its k_eval_trie launches) from an ncu CSV.

    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
        -k regex:k_eval_trie -c K --csv --log-file X.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu
    python scripts/ncu_traffic.py X.csv M > profiles/eval_kernel_ncu.json

K = the number of evaluation launches of one sg_evaluate call (one per level-group range).
bench.py reads the result as roofline.traffic (bytes per sg_evaluate call, ncu-measured).
"""
import csv
import json
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
iname, imet, ival, iid = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per = {}
for r in rows[1:]:
    per.setdefault(r[iid], {"kernel": r[iname]})[r[imet]] = float(r[ival].replace(",", ""))
unit = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
iu = h.index("Metric Unit")
scale = {}
for r in rows[1:]:
    scale[(r[iid], r[imet])] = unit.get(r[iu], 1)
tot_r = sum(v["dram__bytes_read.sum"] * scale[(k, "dram__bytes_read.sum")] for k, v in per.items())
tot_w = sum(v["dram__bytes_write.sum"] * scale[(k, "dram__bytes_write.sum")] for k, v in per.items())
print(json.dumps({"d": 10, "n": 11, "m": int(sys.argv[2]), "launches": len(per),
                  "dram_bytes_read": tot_r, "dram_bytes_write": tot_w,
                  "dram_bytes_per_launch": tot_r + tot_w,
                  "kernels": [v["kernel"][:80] for v in per.values()],
                  "note": "ncu --clock-control none, serialized cold launches; bytes per sg_evaluate call"}, indent=1))
