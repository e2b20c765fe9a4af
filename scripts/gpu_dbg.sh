cd $GRAFT_REPO_ROOT
timeout 300 python -X faulthandler bench.py --log2n 24 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench24.log 2>&1; echo "rc=$?" >> gpurun_out/bench24.log
timeout 300 python -X faulthandler bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench28.log 2>&1; echo "rc=$?" >> gpurun_out/bench28.log
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -k "n2p28 or n2p26 or n2p24" > gpurun_out/pytest_big.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_big.log
