cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"count_kernel" -s 4 -c 1 -o gpurun_out/prof_k2b python scripts/profile_one.py 28 > gpurun_out/ncu4.log 2>&1
