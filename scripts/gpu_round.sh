#!/bin/bash
# One gpurun session with the full evidence set: smoke, GPU tests, the bench line (e2e + cpu baseline),
# the reference arm, the ncu launch list, the DRAM traffic of one evaluation call, ncu --set full captures of
# the group-10 evaluation launches (small-block and large-block) and of the hierarchization, the config
# table, and compute-sanitizer runs.
# Usage (from the repo root, under gpurun --timeout >= 3600): bash scripts/gpu_round.sh TAG
set -x
TAG=${1:-r02}
mkdir -p gpurun_out
nvidia-smi > gpurun_out/${TAG}_nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke exit $?" >> gpurun_out/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/${TAG}_bench.log 2>&1
echo "bench exit $?" >> gpurun_out/${TAG}_bench.log
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_ref.log 2>&1
echo "ref exit $?" >> gpurun_out/${TAG}_bench_ref.log
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/${TAG}_launches.log 2>&1
python scripts/ncu_launches.py gpurun_out/${TAG}_launches.csv > gpurun_out/${TAG}_launches.txt 2>&1
timeout 400 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
  -k regex:k_eval_trie -c 9 --csv --log-file gpurun_out/${TAG}_traffic.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/${TAG}_traffic.log 2>&1
python scripts/ncu_traffic.py gpurun_out/${TAG}_traffic.csv 10000000 > gpurun_out/${TAG}_eval_kernel_ncu.json 2>&1
# group 10: launch 7 = small blocks (R <= 4), launch 8 = large blocks (R >= 5); m = 1e7 (the bench's size)
for L in 7 8; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_eval_trie --launch-skip $L -c 1 \
    -o /tmp/${TAG}_eval_l$L python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/${TAG}_ncu_eval_l$L.log 2>&1
  timeout 120 python scripts/ncu_summary.py /tmp/${TAG}_eval_l$L.ncu-rep > gpurun_out/${TAG}_eval_l${L}_ncu.txt 2>&1
  timeout 120 ncu -i /tmp/${TAG}_eval_l$L.ncu-rep --page source --csv --print-source sass > /tmp/${TAG}_src$L.csv 2>/dev/null
  timeout 120 python scripts/ncu_mix.py /tmp/${TAG}_src$L.csv > gpurun_out/${TAG}_eval_l${L}_mix.txt 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_hier_family -c 2 -o /tmp/${TAG}_hier \
  python bench.py --steps 1 --warmup 0 --m 100000 --no-e2e --no-cpu > gpurun_out/${TAG}_ncu_hier.log 2>&1
timeout 120 python scripts/ncu_summary.py /tmp/${TAG}_hier.ncu-rep > gpurun_out/${TAG}_hier_ncu.txt 2>&1
timeout 600 python scripts/bench_configs.py --reps 5 > gpurun_out/${TAG}_configs.txt 2>&1
# compute-sanitizer is closed on this pool (exit 86, r02v9); the sanitizer driver stays in scripts/sanitize_run.py
# for TOOL in memcheck racecheck initcheck; do
#   timeout 900 compute-sanitizer --tool $TOOL --print-limit 50 python scripts/sanitize_run.py > gpurun_out/${TAG}_sanitizer_$TOOL.txt 2>&1
#   echo "exit $?" >> gpurun_out/${TAG}_sanitizer_$TOOL.txt
# done
ls -la gpurun_out
