# NEXT-1 / NEXT-2 sweep (run under gpurun): their GPU tests, top-k at several
# output sizes on both paths, multi-rank at several m, the multi launch list
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_upper.py tests/test_gpu_multi.py tests/test_gpu_graphs.py -m gpu -x -q > gpurun_out/qc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/qc_pytest.log
for uc in 1048576 16777216 67108864; do
  timeout 300 python bench.py --no-cpu --mode upper --upper-count $uc > gpurun_out/qc_bench_up1_$uc.log 2>&1
  timeout 300 python bench.py --no-cpu --mode upper --upper-count $uc --cfg '{"upper_onepass": 0}' > gpurun_out/qc_bench_up0_$uc.log 2>&1
done
for r in 4 8 16 64; do timeout 300 python bench.py --no-cpu --mode multi --ranks $r > gpurun_out/qc_bench_multi$r.log 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/qc_multi8_launches.csv python bench.py --no-cpu --mode multi --ranks 8 --steps 2 --warmup 3 --e2e-steps 1 > /dev/null 2>&1
