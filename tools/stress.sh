#!/bin/bash
# Repeated runs of the new executions to catch rare races / hangs (under gpurun)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; : > gpurun_out/stress.txt
for r in 1 2 3; do
  timeout 600 python -m pytest tests/test_gpu_dtop.py tests/test_gpu_parity.py -q -x -k "not full_size" >> gpurun_out/stress.txt 2>&1; echo "suite $r rc=$?" >> gpurun_out/stress.txt
done
for d in uniform ascending descending gaussian dups; do
  for k in 64 128 256 512 1024; do
    timeout 120 python tools/dt_case.py 22 $k $d 2 2>&1 | tail -1 | sed "s/^/$d K=$k: /" >> gpurun_out/stress.txt
  done
done
grep -c "sorted=True" gpurun_out/stress.txt; grep -E "HANG|False|rc=[1-9]|Error" gpurun_out/stress.txt | head
