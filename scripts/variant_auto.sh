# DO-BFS bench (C4) for each built variant (build/variants/*) and the default build, R rounds
# interleaved (R=${R:-2}) -> gpurun_out/variants_auto.txt
OUT=gpurun_out/variants_auto.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items() if v['launches']}, d['clocks']['sm_mhz'], d['clocks']['reasons'])"; }
for rep in $(seq 1 ${R:-2}); do
for L in default build/variants/*/libsygraph.so; do
  if [ "$L" = default ]; then unset SYGRAPH_LIB; name=default; else export SYGRAPH_LIB=$L; name=$(basename $(dirname $L)); fi
  python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --dense-roots 0 2>/dev/null | summ "$name" >> $OUT
done
done
sort $OUT
