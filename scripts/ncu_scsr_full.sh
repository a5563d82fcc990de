#!/bin/bash
R=${1:-r01e}
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_push_scsr -s 1 -c 1 \
    -o gpurun_out/${R}_full_scsr python scripts/profile_one_bfs.py push > gpurun_out/${R}_full_scsr.log 2>&1
echo done
