# Quick GPU check of a change (run under gpurun from the repo root):
# the named test files, then a headline bench line and any extra bench args.
#   usage: bash scripts/gpu_quick_check.sh "<pytest files>" ["<bench args>" ...]
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1200 python -m pytest $1 -m gpu -x -q > gpurun_out/qc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/qc_pytest.log
shift
timeout 300 python bench.py --no-cpu > gpurun_out/qc_bench.log 2>&1
i=0
for a in "$@"; do
  i=$((i+1))
  timeout 300 python bench.py --no-cpu $a > gpurun_out/qc_bench_$i.log 2>&1
done
