mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -x -q -k "20 or cfg5" > gpurun_out/s0_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/s0_pytest.log
timeout 300 python scripts/bench_configs.py --reps 5 --only cfg5,cfg2 > gpurun_out/s0_cfg_on.txt 2>&1
SG_TRIE_VAR=Z timeout 300 python scripts/bench_configs.py --reps 5 --only cfg5 > gpurun_out/s0_cfg_off.txt 2>&1
timeout 300 python -m pytest tests -m gpu -x -q > gpurun_out/s0_pytest_all.log 2>&1; echo "pytest exit $?" >> gpurun_out/s0_pytest_all.log
