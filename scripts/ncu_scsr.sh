#!/bin/bash
# launch list (time + DRAM bytes) of one push-only BFS, and a full capture of the level-3 segmented advance
R=${1:-r01c}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_push.csv \
    python scripts/profile_one_bfs.py push > gpurun_out/${R}_one_push.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_push_scsr -s 1 -c 1 \
    -o gpurun_out/${R}_full_scsr python scripts/profile_one_bfs.py push > gpurun_out/${R}_full_scsr.log 2>&1
echo done
