# ncu --set full of the batched-BC cooperative kernels (one 32-source batch of config 5)
ncu --set full --import-source on --clock-control none -k "regex:k_bcb_(forward|backward)" -c 2 \
    -o gpurun_out/bcb_full -f python scripts/profile_bc.py > gpurun_out/ncu_bc.log 2>&1
