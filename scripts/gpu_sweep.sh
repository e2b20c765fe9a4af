cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for b in 64 128 256; do
  timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu --b $b > gpurun_out/bench_b$b.log 2>&1
done
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu --mode approx --b 1024 > gpurun_out/bench_approx1024.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu --mode approx --b 64 > gpurun_out/bench_approx64.log 2>&1
