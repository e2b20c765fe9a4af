cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"sample_tree" -s 6 -c 3 -o gpurun_out/prof_k1 python scripts/profile_one.py 28 > gpurun_out/ncu5.log 2>&1
