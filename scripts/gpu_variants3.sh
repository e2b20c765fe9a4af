cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/var3.log
for v in N G; do
  echo "VARIANT $v" >> gpurun_out/var3.log
  SS_LIB=variants/lib_$v.so timeout 300 python scripts/timeline.py 28 256 2>&1 | grep -E 'L0 K2|per call' >> gpurun_out/var3.log
done
SS_LIB=variants/lib_N.so timeout 600 ncu --set full --clock-control none -k regex:"window_kernel" -s 0 -c 1 -o gpurun_out/k2n python scripts/profile_one.py 28 > gpurun_out/k2n.log 2>&1
