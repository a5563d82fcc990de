# DO and push-only BFS on config 4 for several CTA/grid-tier thresholds (gpurun_out/sweep_heavy.txt)
OUT=gpurun_out/sweep_heavy.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:(round(v['ms'],2),v['launches']) for k,v in d['roofline']['classes'].items()})"; }
for H in 2048 1024 512 256 128; do
  python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --heavy-degree $H 2>/dev/null | summ "auto h=$H" >> $OUT
  python bench.py --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline --direction push --heavy-degree $H 2>/dev/null | summ "push h=$H" >> $OUT
done
