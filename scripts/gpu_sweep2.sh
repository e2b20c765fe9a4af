cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/sw2.log
for cfg in '{}' '{"spec_min_n": 4194304}' '{"spec_min_n": 1048576}' '{"spec_z": 3.0}' '{"spec_z": 3.0, "spec_min_n": 4194304}' '{"spec_min_n": 4194304, "b_deep": 128}'; do
  echo "CFG $cfg" >> gpurun_out/sw2.log
  SS_CFG="$cfg" timeout 300 python scripts/timeline.py 28 256 >> gpurun_out/sw2.log 2>&1
done
