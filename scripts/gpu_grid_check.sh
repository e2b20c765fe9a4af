# small-level window grids: parity subset, multi-rank and headline bench, small-n timelines (under gpurun)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi.py tests/test_gpu_directed.py tests/test_gpu_graphs.py -m gpu -x -q > gpurun_out/qc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/qc_pytest.log
timeout 300 python bench.py --no-cpu > gpurun_out/qc_bench.log 2>&1
for i in 1 2; do timeout 300 python bench.py --no-cpu --mode multi --ranks 8 > gpurun_out/qc_bench_multi8_$i.log 2>&1; done
timeout 300 python bench.py --no-cpu --mode multi --ranks 4 > gpurun_out/qc_bench_multi4.log 2>&1
for L in 16 20 24 28; do timeout 120 python scripts/timeline.py $L 256; done > gpurun_out/qc_tl.log 2>&1
