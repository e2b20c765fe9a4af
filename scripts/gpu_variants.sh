# A/B of library variants built into build_variants/ (run under gpurun):
# headline bench + timeline per variant, the in-tree library first
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for lib in "" build_variants/lib_*.so; do
  name=${lib:-base}; name=$(basename $name .so)
  for rep in 1 2; do
    SS_LIB=$lib timeout 300 python bench.py --no-cpu --steps 50 > gpurun_out/qv_${name}_$rep.log 2>&1
  done
  SS_LIB=$lib timeout 120 python scripts/timeline.py 28 256 > gpurun_out/qv_${name}_tl.log 2>&1
done
