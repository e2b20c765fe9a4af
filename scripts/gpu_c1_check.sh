cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_graphs.py tests/test_gpu_multi.py -m gpu -x -q > gpurun_out/qc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/qc_pytest.log
timeout 300 python bench.py --no-cpu > gpurun_out/qc_bench.log 2>&1
timeout 600 python bench.py --config c1 --steps 10 --warmup 3 > gpurun_out/qc_c1.log 2>&1
for L in 16 17; do timeout 120 python scripts/timeline.py $L 256; done > gpurun_out/qc_tl.log 2>&1
