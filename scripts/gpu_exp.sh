#!/bin/bash
# Experiment runner: bench (with a small oracle parity sample) under several env settings + an ncu capture of the
# group-10 kernel (m = 1e6) each (skip the captures with NCU=0).
# Usage: bash scripts/gpu_exp.sh TAG "ENV1" "ENV2" ...   (each ENV is e.g. "SG_TRIE_VAR=B", or "-" for none)
# ncu reports stay in /tmp on the box (gpurun_out/ must stay < 64 MiB); text summaries come back.
# Every command has its own timeout (<= 8 min per ENV): give gpurun --timeout >= 8 min x #ENV + 5 min.
TAG=$1; shift
mkdir -p gpurun_out
i=0
for E in "$@"; do
  [ "$E" = "-" ] && E=""
  env $E timeout 240 python bench.py --steps 2 --warmup 3 --no-e2e --cpu-budget 3 > gpurun_out/${TAG}_bench$i.log 2>&1
  echo "env=[$E] exit $?" >> gpurun_out/${TAG}_bench$i.log
  if [ "${NCU:-1}" != "0" ]; then
    env $E timeout 240 ncu --set full --clock-control none --import-source on -k regex:k_eval_trie --launch-skip 4 -c 1 -o /tmp/${TAG}_eval$i \
      python bench.py --steps 1 --warmup 0 --m 1000000 --no-e2e --no-cpu > gpurun_out/${TAG}_ncu$i.log 2>&1
    timeout 120 python scripts/ncu_summary.py /tmp/${TAG}_eval$i.ncu-rep > gpurun_out/${TAG}_eval$i.txt 2>&1
    timeout 120 ncu -i /tmp/${TAG}_eval$i.ncu-rep --page source --csv --print-source sass > /tmp/${TAG}_src$i.csv 2>/dev/null
    timeout 120 python scripts/ncu_mix.py /tmp/${TAG}_src$i.csv > gpurun_out/${TAG}_mix$i.txt 2>&1
  fi
  i=$((i+1))
done
echo done
