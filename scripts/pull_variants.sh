# quick DO-BFS bench (config 4) for each built variant (gpurun_out/variants.txt); push-only too if PUSH=1
OUT=gpurun_out/variants.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in r['classes'].items() if v['launches']}, r['kernel'], round(r['frac'],3))"; }
for L in build/variants/*/libsygraph.so; do
  SYGRAPH_LIB=$L python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | summ "$(basename $(dirname $L))" >> $OUT
  if [ "$PUSH" = 1 ]; then SYGRAPH_LIB=$L python bench.py --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline --direction push 2>/dev/null | summ "$(basename $(dirname $L)) push" >> $OUT; fi
done
