#!/bin/bash
# cfg5 experiment (S0 level-0 suffix products + budget-1 closed form vs off) and a Morton lag-cap repeat.
mkdir -p gpurun_out
T=${1:-s1}
timeout 400 python -m pytest tests -m gpu -x -q -k "20 or cfg5" > gpurun_out/${T}_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/${T}_pytest.log
timeout 300 python scripts/bench_configs.py --reps 5 --only cfg5 > gpurun_out/${T}_cfg_on.txt 2>&1
SG_TRIE_VAR=Z timeout 300 python scripts/bench_configs.py --reps 5 --only cfg5 > gpurun_out/${T}_cfg_off.txt 2>&1
timeout 300 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_pytest_all.log 2>&1; echo "pytest exit $?" >> gpurun_out/${T}_pytest_all.log
i=0
for E in ${LAGS:-}; do
  env $E timeout 240 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/${T}_lag$i.log 2>&1
  echo "env=[$E] exit $?" >> gpurun_out/${T}_lag$i.log
  i=$((i+1))
done
