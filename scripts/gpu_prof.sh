#!/bin/bash
# ncu --set full capture of one evaluation launch of the bench workload (default: group 10 at m = 1e7).
# Usage (repo root, under gpurun --timeout >= 900): bash scripts/gpu_prof.sh TAG [M] [SKIP] [REGEX]
#   SKIP = evaluation launches to skip before the captured one (bench step order: groups 0-6, 7, 8, 9, 10).
TAG=${1:-prof}; M=${2:-10000000}; SKIP=${3:-4}; RX=${4:-k_eval}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${RX} --launch-skip ${SKIP} -c 1 \
  -o gpurun_out/${TAG} python bench.py --steps 1 --warmup 0 --m ${M} --no-e2e --no-cpu > gpurun_out/${TAG}_ncu.log 2>&1
echo "ncu exit $?" >> gpurun_out/${TAG}_ncu.log
timeout 120 python scripts/ncu_summary.py gpurun_out/${TAG}.ncu-rep > gpurun_out/${TAG}.txt 2>&1
timeout 120 ncu -i gpurun_out/${TAG}.ncu-rep --page source --csv --print-source sass > /tmp/${TAG}_src.csv 2>/dev/null
timeout 120 python scripts/ncu_mix.py /tmp/${TAG}_src.csv > gpurun_out/${TAG}_mix.txt 2>&1
ls -la gpurun_out/${TAG}*
