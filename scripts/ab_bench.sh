# A/B perf check of env knobs on the C4 BFS bench: bash scripts/ab_bench.sh "SG_X=0" "SG_X=1" ...
OUT=gpurun_out/ab.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items() if v['launches']}, 'frac', round(d['roofline']['frac'],3))"; }
for e in "$@"; do
  env $e python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --dense-roots 0 2>/dev/null | summ "$e" >> $OUT
done
cat $OUT
