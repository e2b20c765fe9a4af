cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 400 -k "not n2p28 and not n2p26 and not n2p24" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
rm -f gpurun_out/tl.log
for a in "28 256 exact 0" "28 64 exact 256" "24 256 exact 0" "28 256 exact 0"; do timeout 300 python scripts/timeline.py $a >> gpurun_out/tl.log 2>&1; done
python scripts/host_overhead.py > gpurun_out/host.log 2>&1
