cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/var4.log
for v in S64 S96 S128; do
  echo "VARIANT $v" >> gpurun_out/var4.log
  SS_LIB=variants/lib_$v.so timeout 300 python scripts/timeline.py 28 256 2>&1 | grep -E 'n=2|L0 K2|per call' >> gpurun_out/var4.log
done
echo "MAIN(160)" >> gpurun_out/var4.log
timeout 300 python scripts/timeline.py 28 256 2>&1 | grep -E 'n=2|L0 K2|per call' >> gpurun_out/var4.log
timeout 600 python -m pytest tests/test_gpu_fused.py -x -q > gpurun_out/fu_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/fu_pytest.log
