cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_upper.py tests/test_gpu_ablation.py -x -q > gpurun_out/up3_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/up3_pytest.log
timeout 300 python bench.py --mode upper --no-cpu > gpurun_out/up3_bench.log 2>&1; echo "rc=$?" >> gpurun_out/up3_bench.log
timeout 300 python bench.py --mode upper --upper-count 134217728 --no-cpu > gpurun_out/up3_bench_half.log 2>&1
timeout 300 python bench.py --mode upper --upper-count 1024 --no-cpu > gpurun_out/up3_bench_small.log 2>&1
timeout 600 python scripts/atomics_ablation.py --out gpurun_out/abl.json > gpurun_out/abl.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"upper_gather" -s 2 -c 1 -o gpurun_out/up3_full python bench.py --mode upper --steps 3 --warmup 3 --no-cpu > gpurun_out/up3_ncu.log 2>&1
