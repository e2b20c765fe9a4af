cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"count_kernel|filter_kernel|sample_tree" -s 9 -c 3 -o gpurun_out/prof2 python scripts/profile_one.py 28 > gpurun_out/ncu2.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu > gpurun_out/bench_b256.log 2>&1
