# QuickSelect partition tiling variants (keys per thread x min CTAs per SM),
# each a separately built libsampleselect.so selected through SS_LIB.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/qpv.log
for lib in paper_conf_ipps_ribizela19_b200/libsampleselect.so _variants/lib_qp_32_3b.so _variants/lib_qp_16_6.so; do
  for dt in float32 float64; do
    echo "LIB $lib $dt" >> gpurun_out/qpv.log
    SS_LIB=$lib timeout 300 python bench.py --mode quick --no-cpu --dtype $dt --steps 30 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['frac'])" >> gpurun_out/qpv.log 2>&1
  done
done
