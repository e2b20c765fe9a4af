# Round evidence: bench line, ncu launch list of the bench command, one full
# capture of the level-0 fused kernel (window_kernel) and of the paper-path
# count/filter kernels, smoke + GPU tests.  Output under gpurun_out/.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/ev_nvsmi.csv
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ev_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/ev_smoke.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/ev_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ev_pytest.log
timeout 600 python bench.py > gpurun_out/ev_bench.log 2>&1; echo "rc=$?" >> gpurun_out/ev_bench.log
timeout 600 python bench.py --mode approx --b 1024 --no-cpu > gpurun_out/ev_bench_approx.log 2>&1
SS_CFG='{"fused_filter": 0}' timeout 300 python scripts/timeline.py 28 256 > gpurun_out/ev_tl_paper.log 2>&1
timeout 300 python scripts/timeline.py 28 256 > gpurun_out/ev_tl.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/ev_ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"window_kernel" -s 0 -c 1 -o gpurun_out/ev_full_w python scripts/profile_one.py 28 > gpurun_out/ev_ncu_full_w.log 2>&1
SS_CFG='{"fused_filter": 0}' timeout 900 ncu --set full --clock-control none --import-source on -k regex:"count_kernel|filter_kernel" -s 0 -c 2 -o gpurun_out/ev_full python scripts/profile_one.py 28 > gpurun_out/ev_ncu_full.log 2>&1
