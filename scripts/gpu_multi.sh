cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multi.py -x -q > gpurun_out/mu_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/mu_pytest.log
timeout 300 python bench.py --mode multi --ranks 8 --steps 20 --no-cpu > gpurun_out/mu_bench_multi8.log 2>&1
timeout 300 python bench.py --mode multi --ranks 32 --steps 10 --no-cpu > gpurun_out/mu_bench_multi32.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/mu_multi_launches.csv python bench.py --mode multi --ranks 8 --steps 2 --warmup 3 --no-cpu > gpurun_out/mu_ncu_multi.log 2>&1
