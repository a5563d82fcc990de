#!/bin/bash
# SCSR (segmented push) check under gpurun: parity tests, then auto / push-only with it on and off.
mkdir -p gpurun_out
OUT=gpurun_out/scsr_check.txt
: > $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "scsr or segmented or tier or config1 or stats" 2>&1 | tail -5 >> $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items()}, 'frac', round(d['roofline']['frac'],3))"; }
for sc in 0 1; do
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --scsr $sc 2>>gpurun_out/scsr_err.txt | summ auto-scsr$sc >> $OUT
  timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --direction push --scsr $sc 2>>gpurun_out/scsr_err.txt | summ push-scsr$sc >> $OUT
done
timeout 600 python -m pytest tests/test_gpu_configs.py -x -q -k "config4" 2>&1 | tail -3 >> $OUT
cat $OUT
