cd $GRAFT_REPO_ROOT
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/ncu_launch_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"count_kernel|filter_kernel|sample_tree" -s 6 -c 3 -o gpurun_out/prof1 python scripts/profile_one.py 28 > gpurun_out/ncu_full.log 2>&1
echo done >> gpurun_out/ncu_full.log
