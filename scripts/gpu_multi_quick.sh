# NEXT-2 quick loop (run under gpurun): multi tests, bench m=4/8/16, ncu brief of the pass
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multi.py -m gpu -x -q > gpurun_out/qc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/qc_pytest.log
for r in 4 8 16; do timeout 300 python bench.py --no-cpu --mode multi --ranks $r > gpurun_out/qc_bench_multi$r.log 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"multi_window_kernel|multi_setup" -c 2 -o gpurun_out/mw_full -f python scripts/profile_one.py 28 multi 8 > gpurun_out/mw_full.log 2>&1
ncu -i gpurun_out/mw_full.ncu-rep --page source --csv -k multi_window_kernel > gpurun_out/mw_source.csv 2>&1
