cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout -s KILL 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu3.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu3.log
: > gpurun_out/c3_gate.jsonl
for k in 128 256 512 1024; do timeout 300 python bench.py --n-log2 26 --K $k --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 >> gpurun_out/c3_gate.jsonl; done
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_w4_gate.log 2>&1; echo "bench rc=$?"
