cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
SS_CFG='{"spec_min_n": 4194304, "spec_z": 3.0}' timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ll.csv python scripts/profile_one.py 28 > gpurun_out/ll.log 2>&1
