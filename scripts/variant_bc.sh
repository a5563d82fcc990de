# C5 batched-BC time per source for each built variant (writes gpurun_out/variants_bc.txt)
OUT=gpurun_out/variants_bc.txt
: > $OUT
for L in build/variants/*/libsygraph.so; do
  SG_TRACE=1 SYGRAPH_LIB=$L python scripts/bench_configs.py --configs 5 --bc-sources 32 > /tmp/v.txt 2>&1
  echo "$(basename $(dirname $L)) $(grep -m1 'batch 0' /tmp/v.txt) $(grep -o '"gpu_ms_per_source": [0-9.]*' /tmp/v.txt)" >> $OUT
done
