#!/bin/bash
# Round-end evidence for the current build (run under gpurun)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout -s KILL 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_w4.log 2>&1; echo "bench rc=$?"
timeout 900 python bench.py --steps 3 --warmup 3 --values --no-cpu-baseline > gpurun_out/bench_w8.log 2>&1; echo "bench w8 rc=$?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.log 2>&1; echo "ref rc=$?"
timeout 600 python bench.py --n-log2 26 --K 128 --dist ascending --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/c3_asc128.log 2>&1; echo "c3 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --profile-steps 2 > /dev/null 2>&1; echo "ncu list rc=$?"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:bgpq_dtop -c 1 -o gpurun_out/prof_dtop -f python bench.py --profile-steps 1 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bgpq_ins_pipe2 -c 1 -o gpurun_out/prof_pipe2 -f python bench.py --profile-steps 1 > gpurun_out/ncu_full2.log 2>&1; echo "ncu full pipe2 rc=$?"
