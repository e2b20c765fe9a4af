cd $GRAFT_REPO_ROOT
timeout 600 python -X faulthandler bench.py "$@" > gpurun_out/bench.log 2>&1; echo "rc=$?" >> gpurun_out/bench.log
