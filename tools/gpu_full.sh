#!/bin/bash
# GPU suite + bench (w=4 and w=8) + ncu launch list of the bench command (under gpurun)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout -s KILL 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_w4.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_w4.log | cut -c1-300
timeout 900 python bench.py --steps 3 --warmup 3 --values --no-cpu-baseline > gpurun_out/bench_w8.log 2>&1; echo "bench w8 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --profile-steps 2 > /dev/null 2>&1; echo "ncu rc=$?"
