#!/bin/bash
# quick SCSR iteration: parity subset, push-only / auto bench with SCSR, launch list of one push-only BFS
R=${1:-r01d}
mkdir -p gpurun_out
OUT=gpurun_out/${R}_scsr.txt
: > $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "scsr or segmented or config1" 2>&1 | tail -3 >> $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items()}, 'frac', round(d['roofline']['frac'],3))"; }
timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>>gpurun_out/${R}_err.txt | summ auto >> $OUT
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --direction push 2>>gpurun_out/${R}_err.txt | summ push >> $OUT
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${R}_launches_push.csv \
    python scripts/profile_one_bfs.py push > /dev/null 2>&1
python scripts/launch_table.py gpurun_out/${R}_launches_push.csv 10 | grep -v "k_scsr_" | tail -40 >> $OUT
cat $OUT
if [ -n "$FULL" ]; then
ncu --set full --clock-control none --import-source on -k regex:k_push_sweep -c 1 \
    -o gpurun_out/${R}_full_sweep python scripts/profile_one_bfs.py push > /dev/null 2>&1
fi
