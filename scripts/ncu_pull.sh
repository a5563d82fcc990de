# ncu --set full of the first pull step of root 0 on config 4 (gpurun_out/pull_full.ncu-rep)
ncu --set full --import-source on --clock-control none -k regex:k_pull_bfs -c 2 \
    -o gpurun_out/pull_full -f python scripts/profile_one_bfs.py auto 0 > gpurun_out/ncu_pull.log 2>&1
