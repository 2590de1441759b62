#!/bin/bash
# ncu --set full capture of the cfg5 (d = 20, n = 6) evaluation kernel, summary + SASS instruction mix.
mkdir -p gpurun_out
T=${1:-cfg5}
timeout 400 ncu --set full --clock-control none --import-source on -k regex:k_eval_trie -c 1 -o /tmp/${T}_eval \
  python scripts/bench_configs.py --reps 1 --only cfg5 > gpurun_out/${T}_ncu.log 2>&1
timeout 120 python scripts/ncu_summary.py /tmp/${T}_eval.ncu-rep > gpurun_out/${T}_eval_ncu.txt 2>&1
timeout 120 ncu -i /tmp/${T}_eval.ncu-rep --page source --csv --print-source sass > /tmp/${T}_src.csv 2>/dev/null
timeout 120 python scripts/ncu_mix.py /tmp/${T}_src.csv > gpurun_out/${T}_eval_mix.txt 2>&1
