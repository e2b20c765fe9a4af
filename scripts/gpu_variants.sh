# A/B of library variants built into build_variants/ (run under gpurun):
# headline bench (twice), a 2^24 bench and the timeline per variant, the
# in-tree library first.  Build a variant with e.g.
#   SS_NVCC_EXTRA="-DSS_WS_CAND=128" python -c "from paper_conf_ipps_ribizela19_b200 import build as b; b.build(out='build_variants/lib_cand128.so')"
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for lib in "" build_variants/lib_*.so; do
  name=${lib:-base}; name=$(basename $name .so)
  for rep in 1 2; do
    SS_LIB=$lib timeout 300 python bench.py --no-cpu --steps 50 > gpurun_out/qv_${name}_$rep.log 2>&1
  done
  SS_LIB=$lib timeout 300 python bench.py --no-cpu --log2n 24 --steps 200 > gpurun_out/qv_${name}_n24.log 2>&1
  SS_LIB=$lib timeout 120 python scripts/timeline.py 28 256 > gpurun_out/qv_${name}_tl.log 2>&1
done
