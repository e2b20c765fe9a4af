# QuickSelect with per-dtype partition occupancy: parity, bench lines, launch list, smoke.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_quick.py -x -q > gpurun_out/q_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/q_pytest.log
timeout 600 python bench.py --mode quick --no-cpu > gpurun_out/q_bench.log 2>&1; echo "rc=$?" >> gpurun_out/q_bench.log
timeout 600 python bench.py --mode quick --no-cpu --dtype float64 > gpurun_out/q_bench64.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/q_launches.csv python bench.py --mode quick --steps 2 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/q_ncu_launch.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/v_smoke.log
