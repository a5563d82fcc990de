# sweep kernel time per variant (ncu launch list, push-only BFS root 0) + push-only bench
OUT=gpurun_out/variants_sweep.txt
: > $OUT
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for L in build/variants/*/libsygraph.so; do
  export SYGRAPH_LIB=$L; name=$(basename $(dirname $L))
  ncu --metrics $M --clock-control none --csv --log-file gpurun_out/v_$name.csv -k regex:k_push_sweep python scripts/profile_one_bfs.py push > /dev/null 2>&1
  echo "$name $(python scripts/launch_table.py gpurun_out/v_$name.csv | grep k_push_sweep | head -1)" >> $OUT
done
unset SYGRAPH_LIB
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3))"; }
if [ -n "$AB" ]; then
for sc in 1 0 1 0; do timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --scsr $sc 2>/dev/null | summ "auto scsr=$sc" >> $OUT; done
fi
cat $OUT
