# Beamer alpha / beta sweep on the C4 DO BFS bench -> gpurun_out/alpha.txt
OUT=gpurun_out/alpha.txt
: > $OUT
for ab in "14 24" "8 24" "20 24" "14 48" "14 96" "8 48" "20 48" "14 24"; do
  set -- $ab
  python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --dense-roots 0 --alpha $1 --beta $2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('alpha $1 beta $2', round(d['value'],1), round(d['ms_per_step'],3), d['per_step'])" >> $OUT
done
cat $OUT
