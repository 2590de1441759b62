#!/bin/bash
# Quick GPU iteration: smoke, parity tests, a short bench, one ncu capture of the group-10 evaluation kernel (m=1e6).
# Usage (under gpurun, from the repo root): bash scripts/gpu_quick.sh TAG [pytest-args]
# Inner timeouts sum to < 25 min: give gpurun --timeout >= 1800.
TAG=${1:-quick}
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/${TAG}_smoke.log
timeout 420 python -m pytest tests -m gpu -x -q ${2:-} > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python bench.py --steps 3 --warmup 3 --no-e2e --cpu-budget 5 > gpurun_out/${TAG}_bench.log 2>&1; echo "bench exit $?" >> gpurun_out/${TAG}_bench.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_eval_trie --launch-skip 4 -c 1 -o gpurun_out/${TAG}_eval \
  python bench.py --steps 1 --warmup 0 --m 1000000 --no-e2e --no-cpu > gpurun_out/${TAG}_ncu_eval.log 2>&1
echo done
