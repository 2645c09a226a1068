#!/bin/bash
# One gpurun call: GPU parity suite + default bench (+ optional extra commands in $EXTRA)
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
timeout -s KILL ${PYTEST_TIMEOUT:-1500} python -u -m pytest tests -m gpu -x -q -p no:cacheprovider --timeout 300 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
if [ -z "$NO_BENCH" ]; then
timeout 600 python bench.py --steps 3 --warmup 3 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
tail -2 gpurun_out/bench.log | cut -c1-1500
fi
if [ -n "$EXTRA" ]; then bash -c "$EXTRA"; fi
