#!/bin/bash
# Round profiling pass (run under gpurun): bench line, ncu launch lists, full captures of the
# dominant kernels; summarised into profiles/ by the commands at the bottom (run locally).
set -u
R=${1:-r02}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,smsp__sass_data_bytes_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum
# 0) the bench line itself (not under a profiler)
timeout 900 python bench.py > gpurun_out/${R}_bench.json 2> gpurun_out/${R}_bench.err
# 1) launch list of the bench command (time only; shares, not absolutes)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${R}_launches_bench.csv \
    python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline --dense-roots 0 --extra-steps 0 > gpurun_out/${R}_ncu_bench.log 2>&1
# 2) one DO BFS and one push-only BFS (host-driven loop): DRAM bytes + LSU sectors per launch
timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_do_dram.csv \
    python scripts/profile_one_bfs.py auto 3 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_push_dram.csv \
    python scripts/profile_one_bfs.py push > /dev/null 2>&1
# 3) full captures (one DO BFS of root index 3: level-2 pull, level-3 pull, late warp pull)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pull_bfs -c 3 \
    -o gpurun_out/${R}_full_pull python scripts/profile_one_bfs.py auto 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_push_sweep -c 1 \
    -o gpurun_out/${R}_full_sweep python scripts/profile_one_bfs.py push > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_bfs_diff -s 2 -c 1 \
    -o gpurun_out/${R}_full_diff python scripts/profile_one_bfs.py auto 0 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_push_heavy -s 2 -c 1 \
    -o gpurun_out/${R}_full_heavy python scripts/profile_one_bfs.py auto 0 > /dev/null 2>&1
# 4) CC (config 3) and SSSP (config 2) kernels, host-driven loops
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pull_ccb -c 1 \
    -o gpurun_out/${R}_full_cc python scripts/profile_one_cc.py 1 host > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k "regex:k_push_words|k_value_diff" -s 4 -c 2 \
    -o gpurun_out/${R}_full_sssp python scripts/profile_one_sssp.py 1 host > /dev/null 2>&1
# 5) every BASELINE config on one GPU (device-resident, next to the oracle)
timeout 1200 python scripts/bench_configs.py > gpurun_out/${R}_configs.jsonl 2> gpurun_out/${R}_configs.err
echo done
# locally:
#   python scripts/make_traffic.py gpurun_out/${R}_launches_do_dram.csv gpurun_out/${R}_launches_push_dram.csv > profiles/traffic.json
#   python scripts/ncu_summary.py gpurun_out/${R}_full_*.ncu-rep > profiles/${R}_ncu_full.txt
#   python scripts/launch_table.py gpurun_out/${R}_launches_do_dram.csv > profiles/${R}_launches_do_dram.txt
