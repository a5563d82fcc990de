python -m pytest tests -m gpu -q -x -k "bc" 2>&1 | tail -2 > gpurun_out/bc_tests.txt
SG_TRACE=1 python scripts/bench_configs.py --configs 5 --bc-sources 32 > gpurun_out/bc_c5.txt 2>&1
