cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"count_kernel" -s 0 -c 1 -o gpurun_out/prof_k2_256 python scripts/profile_one.py 28 exact 256 > gpurun_out/ncu_k2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"count_kernel|filter" -s 0 -c 2 -o gpurun_out/prof_k2_64 python scripts/profile_one.py 28 exact 64 >> gpurun_out/ncu_k2.log 2>&1
