cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"count_kernel" -s 4 -c 1 -o gpurun_out/prof_k2 python scripts/profile_one.py 28 > gpurun_out/ncu3.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"filter_kernel" -s 4 -c 1 -o gpurun_out/prof_k5 python scripts/profile_one.py 28 >> gpurun_out/ncu3.log 2>&1
