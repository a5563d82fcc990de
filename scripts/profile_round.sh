#!/bin/bash
# Round profiling pass (run under gpurun): ncu launch lists + full captures of the dominant kernels,
# summarised into profiles/ by the commands at the bottom (run locally after the merge).
set -u
R=${1:-r01}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed
# 1) launch list of the bench command itself (time only; shares, not absolutes)
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${R}_launches_bench.csv \
    python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline --dense-roots 0 > gpurun_out/${R}_ncu_bench.log 2>&1
# 2) one DO BFS and one push-only BFS (host-driven loop) with DRAM bytes per launch -> traffic.json
ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_do_dram.csv \
    python scripts/profile_one_bfs.py auto > /dev/null 2>&1
ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_push_dram.csv \
    python scripts/profile_one_bfs.py push > /dev/null 2>&1
# 3) full captures: both pull launches (DO), the dense push superstep's sweep (push-only)
ncu --set full --clock-control none --import-source on -k regex:k_pull_bfs -c 2 \
    -o gpurun_out/${R}_full_pull python scripts/profile_one_bfs.py auto > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_push_sweep -c 1 \
    -o gpurun_out/${R}_full_sweep python scripts/profile_one_bfs.py push > /dev/null 2>&1
# 4) the output pass of the dense push level and the level-2 CTA-tier (hub) push (DO)
ncu --set full --clock-control none --import-source on -k regex:k_bfs_diff -s 2 -c 1 \
    -o gpurun_out/${R}_full_diff python scripts/profile_one_bfs.py auto > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_push_heavy -s 2 -c 1 \
    -o gpurun_out/${R}_full_heavy python scripts/profile_one_bfs.py auto > /dev/null 2>&1
echo done
# locally:
#   python scripts/make_traffic.py gpurun_out/${R}_launches_do_dram.csv gpurun_out/${R}_launches_push_dram.csv > profiles/traffic.json
#   python scripts/ncu_summary.py gpurun_out/${R}_full_*.ncu-rep > profiles/${R}_ncu_full.txt
#   python scripts/launch_table.py gpurun_out/${R}_launches_push_dram.csv > profiles/${R}_launches_push_only.txt
