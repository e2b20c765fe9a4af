# NEXT rows: top-k fusion (select_upper), multi-rank selection, atomics ablation.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_upper.py tests/test_gpu_multi.py tests/test_gpu_ablation.py -x -q > gpurun_out/nx_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/nx_pytest.log
timeout 300 python bench.py --mode upper --no-cpu > gpurun_out/nx_bench_upper.log 2>&1
timeout 300 python bench.py --mode upper --upper-count 134217728 --no-cpu > gpurun_out/nx_bench_upper_half.log 2>&1
timeout 300 python bench.py --mode upper --upper-count 1024 --no-cpu > gpurun_out/nx_bench_upper_small.log 2>&1
timeout 300 python bench.py --mode multi --ranks 8 --steps 20 --no-cpu > gpurun_out/nx_bench_multi8.log 2>&1
timeout 300 python bench.py --mode multi --ranks 1 --steps 20 --no-cpu > gpurun_out/nx_bench_multi1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"upper_gather" -s 2 -c 1 -o gpurun_out/nx_upper_full python bench.py --mode upper --steps 3 --warmup 3 --no-cpu > gpurun_out/nx_ncu.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/nx_multi_launches.csv python bench.py --mode multi --ranks 8 --steps 2 --warmup 3 --no-cpu > gpurun_out/nx_ncu_multi.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/nx_pytest_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/nx_pytest_all.log
