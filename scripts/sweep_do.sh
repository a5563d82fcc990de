# Direction-policy sweep on config 4 (writes gpurun_out/sweep.txt)
OUT=gpurun_out/sweep.txt
: > $OUT
summ() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['ms_per_step'],3), {k:round(v['ms'],2) for k,v in d['roofline']['classes'].items() if v['launches']})"; }
for a in ${ALPHAS:-14 40 100 300}; do for b in ${BETAS:-24 8 100}; do
python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --alpha $a --beta $b 2>/dev/null | summ "alpha=$a beta=$b" >> $OUT
done; done
