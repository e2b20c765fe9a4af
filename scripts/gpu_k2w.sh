cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"window_kernel" -s 0 -c 1 -o gpurun_out/k2w python scripts/profile_one.py 28 > gpurun_out/k2w.log 2>&1
