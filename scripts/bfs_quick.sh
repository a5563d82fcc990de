python -m pytest tests -m gpu -q -x -k "bfs or pull or partition or config" 2>&1 | tail -2 > gpurun_out/pull_tests.txt
bash scripts/quick_bench.sh
