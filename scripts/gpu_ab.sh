# A/B bench lines: default vs extra args in $1 (each run -> one JSON line in gpurun_out/ab.log)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/ab.log
for extra in "" "$@"; do
  echo "== $extra" >> gpurun_out/ab.log
  timeout 300 python bench.py --no-cpu --e2e-steps 1 --steps 30 $extra 2>&1 | tail -1 >> gpurun_out/ab.log
done
