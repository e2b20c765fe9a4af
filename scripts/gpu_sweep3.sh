cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/sw3.log
for cfg in '{}' '{"spec_min_n": 4194304}' '{"spec_min_n": 8388608, "spec_z": 3.5}' '{"spec_min_n": 4194304, "spec_z": 3.0}'; do
  echo "CFG $cfg" >> gpurun_out/sw3.log
  SS_CFG="$cfg" timeout 300 python scripts/timeline.py 28 256 >> gpurun_out/sw3.log 2>&1
done
