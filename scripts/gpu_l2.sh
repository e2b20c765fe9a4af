cd $GRAFT_REPO_ROOT
for g in 0 32 64 128; do
  for b in 64 256; do
    echo "== l2fetch=$g b=$b" >> gpurun_out/l2.log
    SS_L2_FETCH=$g timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu --b $b --e2e-steps 1 2>&1 | tail -1 >> gpurun_out/l2.log
  done
done
