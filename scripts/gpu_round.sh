#!/bin/bash
# One gpurun session: GPU tests, smoke, a short bench, the ncu launch list and one full capture.
# Usage (from the repo root, under gpurun): bash scripts/gpu_round.sh TAG [M_PROFILE]
set -x
TAG=${1:-r01}
MP=${2:-1000000}
mkdir -p gpurun_out
nvidia-smi > gpurun_out/${TAG}_nvsmi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke exit $?" >> gpurun_out/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python bench.py --steps 3 --warmup 3 > gpurun_out/${TAG}_bench.log 2>&1
echo "bench exit $?" >> gpurun_out/${TAG}_bench.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/${TAG}_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_eval_trie --launch-skip 4 -c 1 -o gpurun_out/${TAG}_eval \
  python bench.py --steps 1 --warmup 0 --m $MP --no-e2e --no-cpu > gpurun_out/${TAG}_ncu_eval.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_hier -c 2 -o gpurun_out/${TAG}_hier \
  python bench.py --steps 1 --warmup 0 --m 100000 --no-e2e --no-cpu > gpurun_out/${TAG}_ncu_hier.log 2>&1
ls -la gpurun_out
