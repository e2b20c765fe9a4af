cd $GRAFT_REPO_ROOT
for v in build_variants/*.so; do
  for b in 64 256; do
    echo "== $v b=$b" >> gpurun_out/variants.log
    SS_LIB=$PWD/$v timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu --b $b --e2e-steps 1 2>&1 | tail -1 >> gpurun_out/variants.log
  done
done
