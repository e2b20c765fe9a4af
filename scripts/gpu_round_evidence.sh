# Round evidence (run under gpurun from the repo root): smoke, the GPU suite,
# the bench lines (headline + BASELINE configs 1-4 + the paper's level +
# NEXT rows + rotating buffers), the ncu launch list of the bench command,
# full captures of the top kernels, compute-sanitizer runs.  Output under
# gpurun_out/ev_*; copy what is judged to profiles/.
#   usage: bash scripts/gpu_round_evidence.sh [part...]
#   parts: smoke tests bench configs ncu sanitize (default) and next small (NEXT-1/NEXT-2 sweeps,
#   small-n device timelines)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
parts="${*:-smoke tests bench configs ncu sanitize}"
has() { case " $parts " in *" $1 "*) return 0;; esac; return 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw,temperature.gpu --format=csv > gpurun_out/ev_nvsmi.csv
if has smoke; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ev_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/ev_smoke.log
fi
if has tests; then
  timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/ev_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ev_pytest.log
fi
if has bench; then
  timeout 600 python bench.py > gpurun_out/ev_bench.log 2>&1; echo "rc=$?" >> gpurun_out/ev_bench.log
  timeout 300 python bench.py --fused 0 --no-cpu > gpurun_out/ev_bench_paper.log 2>&1
  timeout 300 python bench.py --rotate 9 --no-cpu --steps 45 > gpurun_out/ev_bench_rotate.log 2>&1
  for b in 64 256 1024; do timeout 300 python bench.py --mode approx --b $b --no-cpu > gpurun_out/ev_bench_approx_b$b.log 2>&1; done
  timeout 300 python bench.py --mode upper --no-cpu > gpurun_out/ev_bench_upper.log 2>&1
  timeout 300 python bench.py --mode multi --ranks 8 --no-cpu > gpurun_out/ev_bench_multi8.log 2>&1
  timeout 300 python bench.py --mode quick --no-cpu > gpurun_out/ev_bench_quick.log 2>&1
  timeout 300 python bench.py --dtype float64 --log2n 27 --no-cpu > gpurun_out/ev_bench_f64.log 2>&1
  timeout 300 python scripts/timeline.py 28 256 > gpurun_out/ev_tl.log 2>&1
  SS_CFG='{"fused_filter": 0}' timeout 300 python scripts/timeline.py 28 256 > gpurun_out/ev_tl_paper.log 2>&1
fi
if has configs; then
  for c in c1 c2 c3 c4; do timeout 900 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/ev_config_$c.log 2>&1; done
fi
if has ncu; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/ev_ncu_launch.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"window_kernel|wsel_cluster" -s 0 -c 7 \
    -o gpurun_out/ev_full_fused python scripts/profile_one.py 28 > gpurun_out/ev_ncu_full_fused.log 2>&1
  SS_CFG='{"fused_filter": 0}' timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"count_kernel|filter_kernel" -s 0 -c 2 -o gpurun_out/ev_full_paper python scripts/profile_one.py 28 \
    > gpurun_out/ev_ncu_full_paper.log 2>&1
fi
if has next; then
  # NEXT-1 top-k on both paths at several output sizes; NEXT-2 at several m; its launch list
  for uc in 1048576 16777216 67108864 134217728; do
    timeout 300 python bench.py --no-cpu --mode upper --upper-count $uc > gpurun_out/ev_next_up1_$uc.log 2>&1
    timeout 300 python bench.py --no-cpu --mode upper --upper-count $uc --cfg '{"upper_onepass": 0}' \
      > gpurun_out/ev_next_up0_$uc.log 2>&1
  done
  for r in 4 8 16 64; do timeout 300 python bench.py --no-cpu --mode multi --ranks $r > gpurun_out/ev_next_multi$r.log 2>&1; done
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_next_multi8_launches.csv \
    python bench.py --no-cpu --mode multi --ranks 8 --steps 2 --warmup 3 --e2e-steps 1 > /dev/null 2>&1
fi
if has small; then
  # device timelines (profile = 3 stamps) of small selections and of the approximate variant
  for L in 16 20 24 28; do timeout 120 python scripts/timeline.py $L 256; done > gpurun_out/ev_small_tl.log 2>&1
  # phase stamps (K1w of level 0, the level-1 window) from a stamped build of the library
  SS_NVCC_EXTRA=-DSS_PHASE_STAMPS=1 python -c "from paper_conf_ipps_ribizela19_b200 import build as b; b.build(out='build/lib_stamps.so')" \
    > gpurun_out/ev_small_stamps_build.log 2>&1
  for L in 24 28; do SS_LIB=build/lib_stamps.so WS_DEBUG=1 TL_DEBUG=1 timeout 120 python scripts/timeline.py $L 256; done \
    >> gpurun_out/ev_small_tl.log 2>&1
  for b in 256 1024; do timeout 120 python scripts/timeline.py 28 $b approx; done >> gpurun_out/ev_small_tl.log 2>&1
fi
if has sanitize; then
  nvcc -O2 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include -o build/sanitize_driver scripts/sanitize_driver.cu \
    -Lpaper_conf_ipps_ribizela19_b200 -lsampleselect -Xlinker -rpath="$PWD/paper_conf_ipps_ribizela19_b200" \
    > gpurun_out/ev_san_build.log 2>&1
  timeout 600 build/sanitize_driver > gpurun_out/ev_san_plain.log 2>&1; echo "rc=$?" >> gpurun_out/ev_san_plain.log
  for tool in memcheck racecheck synccheck initcheck; do
    timeout 1200 compute-sanitizer --tool $tool --print-limit 50 build/sanitize_driver 20000 \
      > gpurun_out/ev_san_$tool.log 2>&1; echo "rc=$?" >> gpurun_out/ev_san_$tool.log
  done
fi
