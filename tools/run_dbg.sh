cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for a in "512 drained 173 256" "512 drained 173 0" "512 full 173 0" "512 drained 0 0" "512 drained 499 0"; do
  timeout -s KILL 90 python tools/mixed_debug.py $a > gpurun_out/dbg_"${a// /_}".log 2>&1; echo "$a rc=$?"; tail -2 gpurun_out/dbg_"${a// /_}".log
done
