cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_fused.py -x -q > gpurun_out/fu_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/fu_pytest.log
timeout 300 python scripts/timeline.py 28 1024 approx > gpurun_out/fu_tl.log 2>&1
timeout 300 python scripts/timeline.py 28 256 approx >> gpurun_out/fu_tl.log 2>&1
timeout 300 python scripts/timeline.py 28 64 approx >> gpurun_out/fu_tl.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/fu_pytest2.log 2>&1; echo "rc=$?" >> gpurun_out/fu_pytest2.log
