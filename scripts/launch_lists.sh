#!/bin/bash
# Per-launch time + DRAM bytes of one host-driven BFS on config 4, DO and push-only (run under gpurun).
R=${1:-r01b}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for mode in auto push; do
  ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_${mode}.csv \
      python scripts/profile_one_bfs.py $mode > gpurun_out/${R}_one_${mode}.log 2>&1
done
echo done
