#!/bin/bash
# One `ncu --set full` capture of a kernel (replaces the per-kernel round-1 ncu_*.sh scripts).
#   bash scripts/ncu_full.sh NAME KERNEL_REGEX SKIP COUNT -- python scripts/profile_one_bfs.py auto 0
# -> gpurun_out/NAME.ncu-rep (+ NAME.log).  Read it here with
#    ncu -i gpurun_out/NAME.ncu-rep --page raw --csv   (scripts/ncu_summary.py summarises it)
set -u
NAME=$1; REGEX=$2; SKIP=$3; COUNT=$4; shift 5
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k "regex:${REGEX}" -s "$SKIP" -c "$COUNT" \
    -o "gpurun_out/${NAME}" -f "$@" > "gpurun_out/${NAME}.log" 2>&1
echo "ncu rc=$?"
