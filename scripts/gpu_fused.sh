cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python scripts/timeline.py 28 256 > gpurun_out/fu_tl.log 2>&1
timeout 300 python scripts/timeline.py 24 256 >> gpurun_out/fu_tl.log 2>&1
timeout 300 python scripts/host_overhead.py > gpurun_out/fu_host.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/fu_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/fu_pytest.log
timeout 600 python bench.py --no-cpu --e2e-steps 2 > gpurun_out/fu_bench.log 2>&1
