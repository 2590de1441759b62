#!/bin/bash
# Experiment runner: bench under several env settings + full-size ncu of the group-10 kernel.
# Usage: bash scripts/gpu_exp.sh TAG "ENV1" "ENV2" ...   (each ENV is e.g. "SG_TRIE_MINB=2", or "-" for none)
TAG=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
i=0
for E in "$@"; do
  [ "$E" = "-" ] && E=""
  env $E timeout 600 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/${TAG}_bench$i.log 2>&1
  echo "env=[$E] exit $?" >> gpurun_out/${TAG}_bench$i.log
  env $E timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_eval_trie --launch-skip 4 -c 1 -o gpurun_out/${TAG}_eval$i \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/${TAG}_ncu$i.log 2>&1
  i=$((i+1))
done
echo done
