# A/B of the current build against the one in tmp_v1/ on the same box (under gpurun)
cd "$GRAFT_REPO_ROOT"
for r in 1 2 3; do
  echo "new: $(timeout 300 python tools/pipe_timers.py 27 2>&1 | grep 'insert ms')"
  echo "old: $(cd tmp_v1 && timeout 300 python ../tools/pipe_timers.py 27 2>&1 | grep 'insert ms')"
done
