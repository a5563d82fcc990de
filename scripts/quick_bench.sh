# quick perf check (writes gpurun_out/quick.txt)
OUT=gpurun_out/quick.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items()}, 'frac', round(d['roofline']['frac'],3))"; }
python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | summ auto >> $OUT
python bench.py --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline --direction push 2>/dev/null | summ push-only >> $OUT
