# run quick bench (auto + push-only) for each built variant (writes gpurun_out/variants.txt)
OUT=gpurun_out/variants.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items() if v['launches']})"; }
for L in build/variants/*/libsygraph.so default; do
  if [ "$L" = default ]; then unset SYGRAPH_LIB; name=default; else export SYGRAPH_LIB=$L; name=$(basename $(dirname $L)); fi
  python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | summ "$name auto" >> $OUT
  python bench.py --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline --direction push 2>/dev/null | summ "$name push" >> $OUT
done
