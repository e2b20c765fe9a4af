# NEXT-3 QuickSelect baseline: GPU parity tests, bench lines, ncu launch list,
# one full capture of the level-0 partition kernel.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_quick.py -x -q > gpurun_out/q_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/q_pytest.log
timeout 600 python bench.py --mode quick --no-cpu > gpurun_out/q_bench.log 2>&1; echo "rc=$?" >> gpurun_out/q_bench.log
timeout 600 python bench.py --mode quick --no-cpu --dtype float64 > gpurun_out/q_bench64.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/q_launches.csv python bench.py --mode quick --steps 2 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/q_ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"qs_partition_kernel" -s 0 -c 1 -o gpurun_out/q_full_part python bench.py --mode quick --steps 1 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/q_ncu_full.log 2>&1
