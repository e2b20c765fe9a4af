cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python scripts/dbg_fused.py > gpurun_out/dbg.log 2>&1
timeout 300 python scripts/timeline.py 28 256 > gpurun_out/fu_tl.log 2>&1
timeout 600 python -m pytest tests/test_gpu_fused.py -x -q > gpurun_out/fu_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/fu_pytest.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/fu_pytest2.log 2>&1; echo "rc=$?" >> gpurun_out/fu_pytest2.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"window_kernel" -s 0 -c 1 -o gpurun_out/k2w python scripts/profile_one.py 28 > gpurun_out/k2w.log 2>&1
