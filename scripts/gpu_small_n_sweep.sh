# Latency of small selections (BASELINE c1/c2 sizes): device timelines and
# per-call times for level-0 sample sizes (run under gpurun)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for L in 16 20 24; do
  for s in 0 4096 8192; do
    if [ $s = 0 ]; then cfg='{}'; else cfg="{\"sample_size\": $s}"; fi
    echo "### log2n=$L cfg=$cfg"
    SS_CFG="$cfg" timeout 120 python scripts/timeline.py $L 256 2>&1 | tail -12
  done
done > gpurun_out/qc_small_n.log 2>&1
for L in 28; do
  for b in 256 1024; do
    echo "### approx log2n=$L b=$b"
    timeout 120 python scripts/timeline.py $L $b approx 2>&1 | tail -12
  done
done >> gpurun_out/qc_small_n.log 2>&1
for i in 1 2 3; do timeout 300 python bench.py --no-cpu --mode multi --ranks 8 > gpurun_out/qc_bench_multi8_$i.log 2>&1; done
nvcc -O2 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include -o build/sanitize_driver scripts/sanitize_driver.cu \
  -Lpaper_conf_ipps_ribizela19_b200 -lsampleselect -Xlinker -rpath="$PWD/paper_conf_ipps_ribizela19_b200" > gpurun_out/qc_san_build.log 2>&1
timeout 600 build/sanitize_driver > gpurun_out/qc_san_plain.log 2>&1; echo "rc=$?" >> gpurun_out/qc_san_plain.log
timeout 600 build/sanitize_driver 20000 >> gpurun_out/qc_san_plain.log 2>&1; echo "rc=$?" >> gpurun_out/qc_san_plain.log
