# run quick bench for each built variant (writes gpurun_out/variants.txt)
OUT=gpurun_out/variants.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items() if v['launches']})"; }
for L in build/variants/*/libsygraph.so; do
SYGRAPH_LIB=$L python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | summ $(basename $(dirname $L)) >> $OUT
done
python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | summ default >> $OUT
