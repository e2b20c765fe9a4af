cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/var2.log
for v in A B C D E F; do
  echo "VARIANT $v" >> gpurun_out/var2.log
  SS_LIB=variants/lib_$v.so timeout 300 python scripts/timeline.py 28 256 2>&1 | grep -E 'L0 K2|per call' >> gpurun_out/var2.log
  SS_LIB=variants/lib_$v.so SS_CFG='{"spec_z": 3.0}' timeout 300 python scripts/timeline.py 28 256 2>&1 | grep -E 'L0 K2|per call' >> gpurun_out/var2.log
done
