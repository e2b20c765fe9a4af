cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"filter_kernel|count_kernel" -s 0 -c 4 -o gpurun_out/prof_k5 python scripts/profile_one.py 28 > gpurun_out/ncu_k5.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"sample_rank|sample_tree" -s 0 -c 3 -o gpurun_out/prof_k1 python scripts/profile_one.py 28 > gpurun_out/ncu_k1.log 2>&1
