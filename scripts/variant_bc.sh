OUT=gpurun_out/variants_bc.txt
: > $OUT
for L in build/variants/*/libsygraph.so; do
  SYGRAPH_LIB=$L python scripts/bench_configs.py --configs 5 --bc-sources 32 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$(basename $(dirname $L))', round(d['gpu_ms_per_source'],2), d['supersteps'])" >> $OUT
done
