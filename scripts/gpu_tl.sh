cd $GRAFT_REPO_ROOT
for a in "28 256" "28 128" "28 64" "24 256" "20 256"; do timeout 300 python scripts/timeline.py $a >> gpurun_out/tl.log 2>&1; done
timeout 300 python scripts/timeline.py 28 1024 approx >> gpurun_out/tl.log 2>&1
timeout 300 python scripts/timeline.py 28 256 approx >> gpurun_out/tl.log 2>&1
