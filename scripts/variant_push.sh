# push-only (and optionally auto) bench for each built variant: gpurun_out/variants_push.txt
OUT=gpurun_out/variants_push.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items() if v['launches']})"; }
for L in build/variants/*/libsygraph.so; do
  export SYGRAPH_LIB=$L; name=$(basename $(dirname $L))
  timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --direction push 2>>gpurun_out/variants_err.txt | summ "$name push" >> $OUT
  if [ -n "$AUTO" ]; then timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>>gpurun_out/variants_err.txt | summ "$name auto" >> $OUT; fi
done
cat $OUT
