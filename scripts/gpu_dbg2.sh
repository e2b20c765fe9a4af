cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python scripts/dbg_fused.py > gpurun_out/dbg.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"count_kernel" -s 0 -c 1 -o gpurun_out/k2spec python scripts/profile_one.py 28 > gpurun_out/k2spec.log 2>&1
